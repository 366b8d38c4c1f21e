"""Time the host-to-host paths on C2 (S=128): set_bodies_host + eval_host vs
eval_host_pipelined with several piece counts (wall clock, pinned buffers).
  python tools/e2e_probe.py [--reps 10]"""
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
ap.add_argument("--reps", type=int, default=10)
ap.add_argument("--config", default="C2")
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
inter = h.eval(*[torch.empty(n, device="cuda") for _ in range(4)], stats=True)["interactions_total"]


def timeit(fn):
    fn()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(a.reps):
        fn()
    torch.cuda.synchronize()
    return (time.perf_counter() - t0) / a.reps * 1e3


res = {}
res["host_sequential"] = timeit(lambda: (h.set_bodies(*hx), h.eval(*ho)))
for P in [int(v) for v in os.environ.get("PIECES", "1,2,4,8,16,32").split(",")]:
    res[f"pipelined_{P}"] = timeit(lambda: h.eval_host_pipelined(*hx, *ho, pieces=P))
    res[f"pipelined_{P}_kernel_span_ms"] = h.stats()["kernel_ms"]
res["kernel_only"] = timeit(lambda: h.eval(*[bod[0], bod[1], bod[2], bod[3]]) if False else
                            h.eval(*[torch.empty(0)] * 0) if False else None) if False else None
d = [torch.empty(n, device="cuda") for _ in range(4)]
res["device_eval"] = timeit(lambda: h.eval(*d))
print({k: (round(v, 4) if isinstance(v, float) else v) for k, v in res.items()})
print({k: round(inter / (v * 1e-3) / 1e12, 3) for k, v in res.items() if isinstance(v, float) and "span" not in k},
      "e12 interactions/s")
