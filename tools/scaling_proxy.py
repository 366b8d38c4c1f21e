"""Strong-scaling proxy on ONE GPU: the compute part of an N-GPU run.

Every rank's P2P work is independent (disjoint target leaves, replicated
sources), so rank r of a world-W partition can be timed alone on one GPU: its
kernel time is what GPU r would take.  Reports, per W, the kernel time of every
rank after the library's incremental rebalance from measured times (L18 SIV.D,
as bench.py's warm-up does), and E_W = T_1 / (W * max_r T_r) -- the parallel
efficiency of the kernel alone (no broadcast / gather / launch overheads).

  python tools/scaling_proxy.py --config C2 [--S 128] [--worlds 2,4,8]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_overmanpmm13_b200 as afmm  # noqa: E402
import synth  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--S", type=int, default=None)
    ap.add_argument("--worlds", default="2,4,8")
    ap.add_argument("--rebalance", type=int, default=3)
    a = ap.parse_args()
    c = synth.CONFIGS[a.config]
    S = a.S or c["S"]
    x, y, z, m = synth.make(a.config)
    n = x.shape[0]
    dev = torch.device("cuda", 0)
    st = torch.cuda.Stream(dev)
    torch.cuda.set_stream(st)
    X, Y, Z, M = (torch.from_numpy(v).to(dev) for v in (x, y, z, m))
    tr = afmm.GpuTree(0, stream=st.cuda_stream)
    tr.build(X, Y, Z, S)
    T = tr.copy_out(n)
    b = torch.empty((4, n), device=dev)
    for i, s in enumerate((X, Y, Z, M)):
        tr.gather(s, b[i])
    out = torch.empty((4, n), device=dev)

    def timed(h, reps=20):
        for _ in range(5):
            h.eval(out[0], out[1], out[2], out[3])
        for _ in range(reps):
            h.eval(out[0], out[1], out[2], out[3])
        return float(np.median(h.kernel_times(reps)))

    def handles(W):
        hs = []
        for r in range(W):
            h = afmm.P2P(device=0, rank=r, world=W, eps2=c["eps2"], stream=st.cuda_stream)
            h.set_bodies(b[0], b[1], b[2], b[3])
            h.set_tree(T["leaf_start"], T["leaf_count"], T["u_off"], T["u_idx"])
            hs.append(h)
        return hs

    h1 = handles(1)[0]
    t1 = timed(h1)
    inter = h1.stats()["interactions_total"]
    h1.close()
    res = {"config": a.config, "S": S, "n": n, "interactions": inter, "T1_ms": t1, "worlds": {}}
    for W in [int(v) for v in a.worlds.split(",")]:
        hs = handles(W)
        hist = []
        for it in range(a.rebalance + 1):
            ts = [timed(h) for h in hs]
            hist.append({"max_ms": max(ts), "mean_ms": float(np.mean(ts)),
                         "E": t1 / (W * max(ts)), "tasks": [h.stats()["n_work_items"] for h in hs]})
            if it < a.rebalance:
                for h in hs:
                    h.rebalance(np.array(ts), 0.02)
        res["worlds"][W] = {"rank_ms": [round(t, 4) for t in ts], "history": hist}
        print(f"W={W}: E={hist[-1]['E']:.3f} (first cut {hist[0]['E']:.3f}); rank ms {[round(t, 4) for t in ts]}",
              flush=True)
        for h in hs:
            h.close()
    print(json.dumps(res))


if __name__ == "__main__":
    main()
