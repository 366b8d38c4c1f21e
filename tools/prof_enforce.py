"""Run a few C5 steps' tree maintenance (Enforce_S) for ncu captures of the tree kernels.
  python tools/prof_enforce.py [--n 1048576] [--steps 3]"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_ipps_overmanpmm13_b200 as afmm  # noqa: E402
import synth  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--n", type=int, default=1 << 20)
ap.add_argument("--steps", type=int, default=3)
ap.add_argument("--S", type=int, default=128)
a = ap.parse_args()
x, y, z, m, vx, vy, vz = synth.colliding_with_velocities(a.n, 5)
dom = synth.c5_domain(x, y, z)
dev = torch.device("cuda", 0)
P = [torch.from_numpy(v).to(dev) for v in (x, y, z)]
V = [torch.from_numpy(v).to(dev) for v in (vx, vy, vz)]
t = afmm.GpuTree(0)
t.build(*P, a.S, domain=dom)
for _ in range(a.steps):
    perm = torch.from_numpy(t.copy_out(a.n)["perm"]).long().to(dev)
    P = [p[perm] + 0.05 * v[perm] for p, v in zip(P, V)]
    V = [v[perm] for v in V]
    t.enforce(*P, a.S)
torch.cuda.synchronize()
print("enforce steps done", t.info()["n_leaves"])
