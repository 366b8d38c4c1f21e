"""A/B timing of library builds on one GPU (kernel-only interactions/s on C2).

  python tools/ab.py [--S 32,128,512] [--reps 2] lib1.so lib2.so ...

Each (rep, lib) runs in its own process: the tree for every S is built once,
then the kernel is warmed up for ~0.3 s (clocks ramp up) and timed over 3 x 60
evaluations (median of each block, the best block reported).  Libraries are
interleaved so slow clock drift hits every variant alike."""
import argparse
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = r"""
import sys, os, json, time
sys.path.insert(0, %(root)r)
import numpy as np, torch
import paper_conf_ipps_overmanpmm13_b200 as afmm, synth
try:
    import pynvml; pynvml.nvmlInit(); hnd = pynvml.nvmlDeviceGetHandleByIndex(0)
except Exception:
    hnd = None
x, y, z, m = synth.make(%(config)r)
n = x.shape[0]
dev = torch.device("cuda", 0)
st = torch.cuda.Stream(dev); torch.cuda.set_stream(st)
X, Y, Z, M = (torch.from_numpy(v).to(dev) for v in (x, y, z, m))
res = {}
for S in %(S)r:
    t = afmm.GpuTree(0, stream=st.cuda_stream)
    t.build(X, Y, Z, S)
    T = t.copy_out(n)
    b = torch.empty((4, n), device=dev)
    for i, s in enumerate((X, Y, Z, M)):
        t.gather(s, b[i])
    h = afmm.P2P(eps2=1e-6, stream=st.cuda_stream)
    h.set_bodies(b[0], b[1], b[2], b[3])
    h.set_tree(T["leaf_start"], T["leaf_count"], T["u_off"], T["u_idx"])
    out = torch.empty((4, n), device=dev)
    t0 = time.time()
    while time.time() - t0 < 0.3:
        for _ in range(20):
            h.eval(out[0], out[1], out[2], out[3])
        torch.cuda.synchronize()
    best = 0.0; clk = []
    for blk in range(3):
        for _ in range(60):
            h.eval(out[0], out[1], out[2], out[3])
        if hnd is not None:
            clk.append(pynvml.nvmlDeviceGetClockInfo(hnd, pynvml.NVML_CLOCK_SM))
        km = h.kernel_times(60)
        ips = h.stats()["interactions_total"] / (np.median(km) * 1e-3)
        best = max(best, ips)
    res[S] = (best, clk)
    h.close(); t.close()
print("RESULT", json.dumps(res))
"""


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--S", default="32,128,512", help="comma-separated leaf capacities")
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("--config", default="C2")
    ap.add_argument("libs", nargs="+")
    a = ap.parse_args()
    code = CHILD % {"root": ROOT, "config": a.config, "S": [int(v) for v in a.S.split(",")]}
    table = {}
    for rep in range(a.reps):
        for lib in a.libs:
            # "path.so::K=V,K2=V2" runs that library with extra environment variables
            path, _, kv = lib.partition("::")
            env = dict(os.environ, AFMM_LIB_OVERRIDE=os.path.abspath(path))
            for item in filter(None, kv.split(",")):
                k, _, v = item.partition("=")
                env[k] = v
            r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True, timeout=600)
            line = [ln for ln in r.stdout.splitlines() if ln.startswith("RESULT")]
            if not line:
                print(lib, "FAILED", r.stderr[-800:])
                continue
            import json
            res = json.loads(line[0][7:])
            for S, (ips, clk) in res.items():
                table.setdefault((lib, S), []).append(ips)
                print(f"rep{rep} {lib:50s} S={S:>4s} {ips:.4e} int/s  clk={clk}", flush=True)
    print("\nbest over reps:")
    for (lib, S), v in sorted(table.items(), key=lambda kv: (int(kv[0][1]), kv[0][0])):
        print(f"S={S:>4s} {lib:50s} {max(v):.4e}  ({100 * max(v) * 20 / 74.45e12:.1f}% FP32 peak)")


if __name__ == "__main__":
    main()
