"""Small end-to-end run for compute-sanitizer (memcheck / racecheck / synccheck):
GPU tree (fresh + Enforce_S), device ingest, P2P eval (gravity + Stokeslet),
peer windows, pipelined host evaluation; round 2: rebalance re-ingest, the
caller-driven chunked replication, the serial fallback of the pipelined
evaluation, and (SAN_COMM=1) the library communicator.
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
# round 2: rebalance re-ingesting the handle's copy of a device-ingested tree
h2 = afmm.P2P(eps2=1e-6, world=2, rank=1)
h2.set_bodies(b[0], b[1], b[2], b[3])
h2.set_tree_device(info["n_leaves"], d["leaf_start"], d["leaf_count"], d["u_off"], d["u_idx"])
h2.eval(out[0], out[1], out[2], out[3])
h2.rebalance([1.0, 1.7], 0.0)
h2.eval(out[0], out[1], out[2], out[3])
# round 2: caller-driven chunked replication (chunk masks, epoch-tagged flag word, bounded waits)
from paper_conf_ipps_overmanpmm13_b200 import dist as pdist  # noqa: E402
rp, rb = h1.bodies_buffer()
src = torch.as_tensor(pdist._DeviceArray(rp, rb), device=dev)
hc = afmm.P2P(eps2=1e-6, world=2, rank=1, stream=torch.cuda.current_stream().cuda_stream)
hc.set_bodies(None, None, None, None, n=n)
hc.set_tree_device(info["n_leaves"], d["leaf_start"], d["leaf_count"], d["u_off"], d["u_idx"])
bounds, order = hc.chunks()
dp, db = hc.bodies_buffer()
dst = torch.as_tensor(pdist._DeviceArray(dp, db), device=dev)
side = torch.cuda.Stream()
side.wait_stream(torch.cuda.current_stream())
hc.eval_chunked(out[0], out[1], out[2], out[3])
with torch.cuda.stream(side):
    dst[4 * n:].copy_(src[4 * n:])
    for j, c in enumerate(order):
        dst[4 * int(bounds[c]):4 * int(bounds[c + 1])].copy_(src[4 * int(bounds[c]):4 * int(bounds[c + 1])])
        hc.publish_chunks(j + 1, side.cuda_stream)
hc.stats()
# round 2: serial fallback of the pipelined evaluation (no co-resident pack block)
os.environ["AFMM_PACK_CORESIDENT"] = "0"
os.environ["AFMM_E2E_ZEROCOPY"] = "1"
hf = afmm.P2P(eps2=1e-6)
hf.set_bodies(b[0], b[1], b[2], b[3])
hf.set_tree(T["leaf_start"], T["leaf_count"], T["u_off"], T["u_idx"])
hf.eval_host_pipelined(*hx, *ho, pieces=1)
if os.environ.get("SAN_COMM") == "1":          # library communicator, one rank (NCCL's own kernels included)
    hn = afmm.P2P(eps2=1e-6, nccl_id=afmm.nccl_id())
    hn.set_bodies(b[0], b[1], b[2], b[3])
    hn.set_tree(T["leaf_start"], T["leaf_count"], T["u_off"], T["u_idx"])
    hn.eval(out[0], out[1], out[2], out[3], stats=True)
    hn.close()
torch.cuda.synchronize()
print("sanitize run ok", info["n_leaves"])
