"""Small end-to-end run for compute-sanitizer (memcheck / racecheck / synccheck):
GPU tree (fresh + Enforce_S), device ingest, P2P eval (gravity + Stokeslet),
peer windows, pipelined host evaluation.
  compute-sanitizer --tool memcheck python tools/sanitize_run.py"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_overmanpmm13_b200 as afmm  # noqa: E402
import synth  # noqa: E402

n = int(os.environ.get("SAN_N", "20000"))
x, y, z, m = synth.make("plummer", n, 3)
dev = torch.device("cuda", 0)
X, Y, Z, M = (torch.from_numpy(v).to(dev) for v in (x, y, z, m))
t = afmm.GpuTree(0)
info = t.build(X, Y, Z, 32)
t.enforce(X * 1.0001, Y, Z, 32)
info = t.build(X, Y, Z, 32)
T = t.copy_out(n)
d = t.device_arrays()
b = torch.empty((4, n), device=dev)
for i, s in enumerate((X, Y, Z, M)):
    t.gather(s, b[i])
rows = torch.empty_like(b)
t.gather_rows(b, rows)
out = torch.empty((4, n), device=dev)
peer = torch.empty((4, n), device=dev)
h = afmm.P2P(eps2=1e-6, world=2, rank=0)
h.set_bodies(b[0], b[1], b[2], b[3])
h.set_tree_device(info["n_leaves"], d["leaf_start"], d["leaf_count"], d["u_off"], d["u_idx"])
h.set_peer_windows([tuple(peer[a] for a in range(4))])
h.eval(out[0], out[1], out[2], out[3])
h.set_peer_windows([])
h1 = afmm.P2P(eps2=1e-6)
h1.set_bodies(b[0], b[1], b[2], b[3])
h1.set_tree(T["leaf_start"], T["leaf_count"], T["u_off"], T["u_idx"])
h1.eval(out[0], out[1], out[2], out[3])
hx = [b[a].cpu().pin_memory() for a in range(4)]
ho = [torch.empty(n).pin_memory() for _ in range(4)]
h1.eval_host_pipelined(*hx, *ho, pieces=3)                 # zero-copy, input chain from its graph
os.environ["AFMM_INPUT_GRAPH"] = "0"
h1.eval_host_pipelined(*hx, *ho, pieces=3)                 # zero-copy, direct launches
os.environ["AFMM_E2E_ZEROCOPY"] = "0"
h1.eval_host_pipelined(*hx, *ho, pieces=3)                 # staged copies + per-piece copy-back
fx, fy, fz = (torch.from_numpy(np.ascontiguousarray(v)).to(dev) for v in synth.uniform_with_forces(n, 4)[3:])
hs = afmm.P2P(eps2=1e-6, law=afmm.LAW_STOKESLET)
hs.set_bodies_stokeslet(b[0], b[1], b[2], fx, fy, fz)
hs.set_tree(T["leaf_start"], T["leaf_count"], T["u_off"], T["u_idx"])
hs.eval(out[0], out[1], out[2], out[3])
torch.cuda.synchronize()
print("sanitize run ok", info["n_leaves"])
