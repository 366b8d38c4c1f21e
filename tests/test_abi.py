"""CPU tests of the C-ABI library: it loads, exports every symbol the headers
declare, and its host-only functions agree with the oracle bit-exactly."""
import ctypes
import os
import re

import numpy as np
import pytest

import oracle
import synth

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    names = []
    for h in ("afmm_p2p.h", "afmm_tree.h", "afmm_step.h", "afmm_balance.h"):
        src = open(os.path.join(ROOT, "include", h)).read()
        src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
        names += re.findall(r"\b(afmm_\w+)\s*\(", src)
    return sorted(set(names))


def test_library_loads_and_exports_every_declared_symbol():
    import paper_conf_ipps_overmanpmm13_b200 as afmm
    lib = ctypes.CDLL(afmm.LIB_PATH)
    decl = _declared()
    assert len(decl) >= 25
    for name in decl:
        assert hasattr(lib, name), name
    assert sorted(afmm.EXPORTED) == decl
    assert "sm_100a" in afmm.version()


def test_library_is_sm100a_cubin():
    import subprocess
    import paper_conf_ipps_overmanpmm13_b200 as afmm
    out = subprocess.run(["cuobjdump", "-lelf", afmm.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


@pytest.mark.parametrize("dist,n,S", [("uniform", 4096, 64), ("plummer", 30000, 32),
                                      ("colliding", 30000, 100)])
def test_interactions_and_literal_partition_bit_exact(dist, n, S):
    import paper_conf_ipps_overmanpmm13_b200 as afmm
    x, y, z, m = synth.make(dist, n, 5)
    T = oracle.Tree(x, y, z, S)
    I_ref = oracle.interactions(T.leaf_count, T.u_off, T.u_idx)
    I = afmm.interactions(T.leaf_count, T.u_off, T.u_idx)
    assert np.array_equal(I, I_ref)
    for G in (1, 2, 3, 4, 8, 16):
        _, split_ref = oracle.partition_literal(I_ref, G)
        assert np.array_equal(afmm.partition_literal(I, G), split_ref)
        # the weighted rule with integer-valued weights gives the same cut
        assert np.array_equal(afmm.partition_weighted(I.astype(np.float64), G), split_ref)


def test_partition_edge_cases():
    import paper_conf_ipps_overmanpmm13_b200 as afmm
    assert list(afmm.partition_literal(np.array([5, 1, 1]), 8)) == [0, 1, 2, 3, 3, 3, 3, 3, 3]
    assert list(afmm.partition_literal(np.array([7]), 1)) == [0, 1]
    assert list(afmm.partition_literal(np.array([1, 1, 1, 1]), 2)) == [0, 2, 4]
    with pytest.raises(afmm.AfmmError):
        afmm.partition_literal(np.array([1, -1]), 2)
    with pytest.raises(afmm.AfmmError):
        afmm.partition_weighted(np.array([1.0, np.nan]), 2)


def test_interactions_rejects_bad_index():
    import paper_conf_ipps_overmanpmm13_b200 as afmm
    with pytest.raises(afmm.AfmmError):
        afmm.interactions(np.array([1, 1]), np.array([0, 1, 2]), np.array([0, 2]))


def test_ctypes_structs_match_the_c_headers(tmp_path):
    """Every ctypes mirror of a header struct has the C layout: the same size and
    the same offset for every field (compiled with gcc against include/*.h), so a
    field added on one side only fails here rather than corrupting calls."""
    import paper_conf_ipps_overmanpmm13_b200 as afmm
    pairs = [("afmm_p2p_config", afmm.Config), ("afmm_p2p_stats", afmm.Stats), ("afmm_ipc_handle", afmm.IpcHandle),
             ("afmm_lb_config", afmm.LbConfig), ("afmm_fg_result", afmm.FgResult)]
    lines = ['#include <stdio.h>', '#include <stddef.h>', '#include "afmm_balance.h"', "int main(void) {"]
    for cname, py in pairs:
        lines.append(f'printf("{cname} size %zu\\n", sizeof({cname}));')
        for f, _ in py._fields_:
            lines.append(f'printf("{cname} {f} %zu\\n", offsetof({cname}, {f}));')
    lines += ["return 0;", "}"]
    src = tmp_path / "layout.c"
    src.write_text("\n".join(lines))
    exe = tmp_path / "layout"
    import subprocess
    subprocess.check_call(["gcc", "-std=c11", "-I", os.path.join(ROOT, "include"), str(src), "-o", str(exe)])
    got = {}
    for ln in subprocess.check_output([str(exe)], text=True).splitlines():
        a, b, v = ln.split()
        got[(a, b)] = int(v)
    for cname, py in pairs:
        assert got[(cname, "size")] == ctypes.sizeof(py), cname
        for f, _ in py._fields_:
            assert got[(cname, f)] == getattr(py, f).offset, (cname, f)


def test_plain_c_caller_builds():
    """examples/c_abi_demo.c -- a C program using only include/*.h and the .so
    (tree builder + host-pointer P2P entry points + stats) -- compiles and links
    with gcc (`make demo`); it runs on the GPU in tests/test_gpu_c_demo.py."""
    import subprocess
    r = subprocess.run(["make", "-C", ROOT, "demo"], capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-2000:]
    assert os.path.exists(os.path.join(ROOT, "examples", "c_abi_demo"))
