"""The plain-C caller (examples/c_abi_demo.c, no Python on its path) on the GPU:
tree build, P2P through the host-pointer entry points, its own fp64 direct-sum
check of 64 sampled leaves; exit status 0 = within 1e-5 per body on phi."""
import os
import subprocess

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize("n,S", [(200000, 64), (50000, 7), (1, 1)])
def test_c_abi_demo_runs(n, S):
    r = subprocess.run(["make", "-C", ROOT, "demo"], capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stderr[-2000:]
    r = subprocess.run([os.path.join(ROOT, "examples", "c_abi_demo"), str(n), str(S)], capture_output=True,
                       text=True, timeout=300)
    assert r.returncode == 0, r.stdout + r.stderr
    assert "phi_max_rel" in r.stdout
