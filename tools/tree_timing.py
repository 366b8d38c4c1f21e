"""Wall time of each tree-maintenance call on the C5 workload (1 M colliding
bodies): a fresh build, then Enforce_S / KEEP rebuilds / edited rebuilds along
a drifting trajectory, each call synchronised and timed on the host, with the
handle's counters.  Diagnostic only (no JSON contract):

  python tools/tree_timing.py [--n 1048576] [--S 360] [--levels]"""
import argparse
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_overmanpmm13_b200 as afmm  # noqa: E402
import synth  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--n", type=int, default=1 << 20)
ap.add_argument("--S", type=int, default=360)
ap.add_argument("--levels", action="store_true", help="force the level loop (AFMM_TREE_LEVELS=1)")
a = ap.parse_args()
if a.levels:
    os.environ["AFMM_TREE_LEVELS"] = "1"
x, y, z, m, vx, vy, vz = synth.colliding_with_velocities(a.n, 5)
dom = synth.c5_domain(x, y, z)
dev = torch.device("cuda", 0)
P = torch.from_numpy(np.stack([x, y, z])).to(dev)
V = torch.from_numpy(np.stack([vx, vy, vz])).to(dev)
bufs = [P.clone(), P.clone()]
t = afmm.GpuTree(0)


def timed(name, fn):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    info = fn()
    torch.cuda.synchronize()
    dt = 1e3 * (time.perf_counter() - t0)
    t1 = time.perf_counter()
    c = t.farfield_counts()
    dc = 1e3 * (time.perf_counter() - t1)
    print(f"{name:28s} {dt:8.3f} ms  L={info['n_leaves']}  {t.counters()}  farfield_counts {dc:.3f} ms {c.tolist()}",
          flush=True)


timed("build S=128", lambda: t.build(P[0], P[1], P[2], 128, domain=dom))
perm = torch.from_numpy(t.copy_out(a.n)["perm"].astype(np.int64)).to(dev)
P, V = P[:, perm].contiguous(), V[:, perm].contiguous()
plan = ["keep"] * 4 + ["enforce"] * 3 + ["keep"] * 6 + ["keep+edits"] * 2 + ["keep"] * 3
rng = np.random.default_rng(1)
for step, op in enumerate(plan):
    P = P + 0.05 * V
    b = bufs[step % 2]
    b.copy_(P)
    if op == "keep":
        timed(f"{step:2d} keep", lambda: t.rebuild(b[0], b[1], b[2], a.S, mode=afmm.TREE_KEEP))
    elif op == "enforce":
        timed(f"{step:2d} enforce S={a.S}", lambda: t.enforce(b[0], b[1], b[2], a.S))
    else:
        nd = t.nodes()
        pick = rng.random(nd["level"].shape[0]) < 0.02
        ed = [(int(l), int(p), 1 if c > 0 else 2) for l, p, c, k in
              zip(nd["level"], nd["prefix"], nd["nchild"], pick) if k]
        timed(f"{step:2d} keep+{len(ed)} edits", lambda: t.rebuild(b[0], b[1], b[2], a.S, mode=afmm.TREE_KEEP,
                                                                     edits=ed))
    perm = torch.from_numpy(t.copy_out(a.n)["perm"].astype(np.int64)).to(dev)
    P, V = P[:, perm].contiguous(), V[:, perm].contiguous()
t.close()
