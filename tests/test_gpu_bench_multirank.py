"""bench.py's N > 1 flow end to end on ONE GPU: two torchrun ranks on the same
device over gloo (AFMM_BENCH_SAME_DEVICE=1, the caller-side path: one broadcast of
the packed bodies, the P2P kernel storing into both ranks' outputs over CUDA-IPC
peer windows, the max over ranks), on the small C1 workload.  Checks the printed
JSON line against the contract (one line on rank 0, n_gpus, strong scaling, the
same config dict as N = 1, launches counted over both ranks).  The NCCL library
communicator needs one GPU per rank and is not exercised here;
no kernel of one rank waits on the other's."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_bench_two_ranks_same_gpu_gloo():
    env = dict(os.environ, AFMM_BENCH_SAME_DEVICE="1", MASTER_ADDR="127.0.0.1")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", "29541", os.path.join(ROOT, "bench.py"),
           "--gpus", "2", "--steps", "3", "--warmup", "3", "--config", "C1", "--dist-backend", "gloo",
           "--no-cpu-baseline"]
    r = subprocess.run(cmd, env=env, capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["steps"] == 3 and d["scaling"] == "strong"
    assert d["value"] > 0 and d["ms_per_step"] > 0 and d["higher_is_better"] is True
    assert d["config"]["name"] == "C1" and d["config"]["parallelism"].endswith("x2 (cost model, PAPER L16)")
    assert d["gpu_launches"] >= 2 * 3                  # at least a P2P launch per rank per timed step
    assert d["e2e"]["value"] > 0


def test_bench_n1_contract_fields():
    """bench.py at N = 1 on the small C1 workload prints one JSON line with every
    key the driver contract names: metric/value/unit, timing, roofline (bound,
    achieved, peak, frac, traffic), cpu_baseline (oracle, cores, sample), e2e with
    the copied bytes, clocks sampled during the timed region, gpu_launches."""
    cmd = [sys.executable, os.path.join(ROOT, "bench.py"), "--config", "C1", "--steps", "3", "--warmup", "3",
           "--no-sweep", "--no-stokeslet", "--no-proxy", "--cpu-seconds", "0.5", "--cpu-seconds-1core", "0.3"]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    d = json.loads(lines[0])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
              "vs_baseline", "dtype", "data", "config", "roofline", "cpu_baseline", "e2e", "clocks", "gpu_launches"):
        assert k in d, k
    assert d["n_gpus"] == 1 and d["steps"] == 3 and d["warmup"] >= 3 and d["value"] > 0
    assert d["unit"] == "interactions/s" and d["higher_is_better"] is True and d["dtype"] == "f32"
    rf = d["roofline"]
    assert rf["bound"] == "alu" and rf["unit"] == "TFLOP/s" and 0 < rf["frac"] < 1
    assert abs(rf["frac"] - rf["achieved"] / rf["peak"]) < 1e-9
    cb = d["cpu_baseline"]
    assert cb["kind"] == "oracle" and cb["cores"] >= 1 and cb["value"] > 0 and cb["sample"]
    e = d["e2e"]
    assert e["value"] > 0 and e["h2d_bytes_per_step"] > 0 and e["d2h_bytes_per_step"] > 0
    assert d["gpu_launches"] >= 3
    assert "sm_mhz" in d["clocks"] and "reasons" in d["clocks"]
    assert d["config"]["name"] == "C1" and d["config"]["workload"]
