"""Run the P2P kernel on one config/S a few times (for ncu captures).

  python tools/prof_p2p.py --config C2 --S 128 --evals 4
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_overmanpmm13_b200 as afmm  # noqa: E402
import synth  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--S", type=int, default=None)
ap.add_argument("--evals", type=int, default=4)
ap.add_argument("--law", default="gravity", choices=["gravity", "stokeslet"])
a = ap.parse_args()
c = synth.CONFIGS[a.config]
S = a.S or c["S"]
if a.law == "stokeslet":
    x, y, z, fx, fy, fz = synth.uniform_with_forces(c["n"], c["seed"])
    m = fx
else:
    x, y, z, m = synth.make(a.config)
n = x.shape[0]
dev = torch.device("cuda", 0)
st = torch.cuda.Stream(dev)
torch.cuda.set_stream(st)
X, Y, Z, M = (torch.from_numpy(v).to(dev) for v in (x, y, z, m))
t = afmm.GpuTree(0, stream=st.cuda_stream)
t.build(X, Y, Z, S)
T = t.copy_out(n)
b = torch.empty((4, n), device=dev)
for i, s in enumerate((X, Y, Z, M)):
    t.gather(s, b[i])
if a.law == "stokeslet":
    F = [torch.from_numpy(v).to(dev) for v in (fx, fy, fz)]
    Fs = torch.empty((3, n), device=dev)
    for i in range(3):
        t.gather(F[i], Fs[i])
    h = afmm.P2P(eps2=c["eps2"], stream=st.cuda_stream, law=afmm.LAW_STOKESLET)
    h.set_bodies_stokeslet(b[0], b[1], b[2], Fs[0], Fs[1], Fs[2])
else:
    h = afmm.P2P(eps2=c["eps2"], stream=st.cuda_stream)
    h.set_bodies(b[0], b[1], b[2], b[3])
h.set_tree(T["leaf_start"], T["leaf_count"], T["u_off"], T["u_idx"])
out = torch.empty((4, n), device=dev)
for _ in range(a.evals):
    h.eval(out[0], out[1], out[2], out[3])
km = h.kernel_times(a.evals)
s = h.stats()
print({"config": a.config, "S": S, "n_leaves": T["n_leaves"], "interactions": s["interactions_total"],
       "kernel_ms": [round(v, 4) for v in km], "int_per_s": s["interactions_total"] / (np.median(km) * 1e-3),
       "items": s["n_work_items"], "buckets": s["bucket_interactions"]})
