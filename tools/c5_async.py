"""The bench's C5 line alone (1 Mi colliding bodies, S = 128, KDK with Enforce_S and
device ingest every step): 5 warm-up steps, then R repeats of 60 back-to-back
steps (sync=False), printing the per-step means of each repeat.  For A/B runs of
library builds (AFMM_LIB_OVERRIDE):  python tools/c5_async.py [R]"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_ipps_overmanpmm13_b200.timeloop import TimeLoop  # noqa: E402

R = int(sys.argv[1]) if len(sys.argv) > 1 else 3
c5 = synth.CONFIGS["C5"]
x, y, z, m, vx, vy, vz = synth.colliding_with_velocities(c5["n"], c5["seed"])
loop = TimeLoop(x, y, z, m, vx, vy, vz, c5["S"], c5["eps2"], 0.05, synth.c5_domain(x, y, z), device=0)
for _ in range(5):
    loop.step()
for rep in range(R):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    recs = [loop.step(sync=False) for _ in range(60)]
    loop.finish(recs)
    wall = 1e3 * (time.perf_counter() - t0) / len(recs)
    keys = ("kernel_ms", "enforce_ms", "set_tree_ms", "gpu_step_ms")
    print(json.dumps({"rep": rep, "step_ms": round(wall, 4),
                      **{k: round(float(np.mean([r[k] for r in recs])), 4) for k in keys}}), flush=True)
loop.close()
