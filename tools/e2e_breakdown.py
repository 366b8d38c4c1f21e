"""Where the host-to-host time goes (C2, S=128): eval_host_pipelined in each
AFMM_E2E_ZEROCOPY mode ("1" both, "i" inputs only, "o" outputs only, "0"
staged) -- wall per call, the GPU span between events recorded on the handle's
stream around the call, and the kernel's own span (stats.kernel_ms).
  python tools/e2e_breakdown.py [--reps 20]"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_ipps_overmanpmm13_b200 as afmm  # noqa: E402
import synth  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--reps", type=int, default=20)
ap.add_argument("--config", default="C2")
ap.add_argument("--pieces", type=int, default=1, help="output pieces (staged-output modes copy each back as it completes)")
ap.add_argument("--modes", default="1,i,o,0")
a = ap.parse_args()
c = synth.CONFIGS[a.config]
x, y, z, m = synth.make(a.config)
n = x.shape[0]
st = torch.cuda.Stream()
torch.cuda.set_stream(st)
X, Y, Z, M = (torch.from_numpy(v).cuda() for v in (x, y, z, m))
t = afmm.GpuTree(0, stream=st.cuda_stream)
t.build(X, Y, Z, c["S"])
T = t.copy_out(n)
bod = torch.empty((4, n), device="cuda")
for i, s in enumerate((X, Y, Z, M)):
    t.gather(s, bod[i])
hx = [bod[i].cpu().pin_memory() for i in range(4)]
ho = [torch.empty(n).pin_memory() for _ in range(4)]
h = afmm.P2P(eps2=c["eps2"], stream=st.cuda_stream)
h.set_bodies(*bod)
h.set_tree(T["leaf_start"], T["leaf_count"], T["u_off"], T["u_idx"])
d = [torch.empty(n, device="cuda") for _ in range(4)]
inter = h.eval(*d, stats=True)["interactions_total"]
res = {"interactions": inter}
for mode in a.modes.split(","):
    os.environ["AFMM_E2E_ZEROCOPY"] = mode
    for _ in range(3):
        h.eval_host_pipelined(*hx, *ho, pieces=a.pieces)
    torch.cuda.synchronize()
    wall, span, kern = [], [], []
    for _ in range(a.reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        t0 = time.perf_counter()
        h.eval_host_pipelined(*hx, *ho, pieces=a.pieces)
        wall.append((time.perf_counter() - t0) * 1e3)
        e1.record(st)
        e1.synchronize()
        span.append(e0.elapsed_time(e1))
        kern.append(h.stats()["kernel_ms"])
    med = lambda v: sorted(v)[len(v) // 2]  # noqa: E731
    res[mode] = {"wall_ms": round(med(wall), 4), "gpu_span_ms": round(med(span), 4), "kernel_ms": round(med(kern), 4),
                 "wall_e12": round(inter / med(wall) / 1e9, 3)}
os.environ["AFMM_E2E_ZEROCOPY"] = "1"
for _ in range(3):
    h.eval(*d)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(st)
for _ in range(a.reps):
    h.eval(*d)
e1.record(st)
e1.synchronize()
res["device_eval_ms"] = round(e0.elapsed_time(e1) / a.reps, 4)
print(json.dumps(res))
