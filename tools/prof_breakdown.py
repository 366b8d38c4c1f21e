"""Per-warp cycle breakdown of the P2P kernel (a -DAFMM_PROF=1 tuning build).

  AFMM_LIB_OVERRIDE=build/var_prof/libafmm_p2p.so python tools/prof_breakdown.py --S 32,128,512

Slots (clock64 deltas summed per warp, see p2p_kernel.cuh PROF_*): issue of the
next chunk, mbarrier wait, task start (targets, zeroing), math (consume), task
end (fold, copy reduction, stores), trailing __syncwarp, whole loop; chunk and
task counts; globaltimer at start / end (tail = how long warps sit idle while
others finish)."""
import argparse
import ctypes as C
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_overmanpmm13_b200 as afmm  # noqa: E402
import synth  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--S", default="32,128,512")
ap.add_argument("--config", default="C2")
ap.add_argument("--warps", type=int, default=12)
a = ap.parse_args()
lib = afmm._lib
lib.afmm_p2p_prof_read.restype = C.c_int
lib.afmm_p2p_prof_read.argtypes = [C.c_void_p, C.c_int]
x, y, z, m = synth.make(a.config)
n = x.shape[0]
dev = torch.device("cuda", 0)
st = torch.cuda.Stream(dev)
torch.cuda.set_stream(st)
X, Y, Z, M = (torch.from_numpy(v).to(dev) for v in (x, y, z, m))
names = ["issue", "wait", "first", "math", "last", "sync"]
for S in [int(v) for v in a.S.split(",")]:
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
    for _ in range(30):
        h.eval(out[0], out[1], out[2], out[3])
    torch.cuda.synchronize()
    nw = 148 * a.warps
    buf = np.zeros(nw * 16, np.uint64)
    lib.afmm_p2p_prof_read(buf.ctypes.data, buf.size)
    P = buf.reshape(nw, 16).astype(np.float64)
    loop = P[:, 8]
    frac = {k: P[:, i].sum() / loop.sum() for i, k in enumerate(names)}
    gt0, gt1 = P[:, 9], P[:, 10]
    span = gt1.max() - gt0.min()
    busy = (gt1 - gt0).sum() / (nw * span)
    km = h.kernel_times(10)
    s = h.stats()
    print(f"S={S}: kernel {np.median(km):.4f} ms, {s['interactions_total'] / (np.median(km) * 1e-3):.3e} int/s; "
          f"chunks/warp {P[:, 6].mean():.1f}, tasks/warp {P[:, 7].mean():.1f}; cycles/chunk {loop.sum() / P[:, 6].sum():.0f}")
    print("   loop cycle shares: " + ", ".join(f"{k} {100 * v:.1f}%" for k, v in frac.items())
          + f", other {100 * (1 - sum(frac.values())):.1f}%")
    print(f"   warp end times: min {(gt1.min() - gt0.min()) / 1e3:.1f} us, median {(np.median(gt1) - gt0.min()) / 1e3:.1f} us, "
          f"max {(gt1.max() - gt0.min()) / 1e3:.1f} us; start skew {(gt0.max() - gt0.min()) / 1e3:.1f} us; "
          f"warp-busy fraction of the span {100 * busy:.1f}%")
    per_task_last = P[:, 4].sum() / P[:, 7].sum()
    per_task_first = P[:, 2].sum() / P[:, 7].sum()
    print(f"   per task: first {per_task_first:.0f} cyc, last {per_task_last:.0f} cyc; per chunk: issue "
          f"{P[:, 0].sum() / P[:, 6].sum():.0f} (meta {P[:, 12].sum() / P[:, 6].sum():.0f}, copies {P[:, 13].sum() / P[:, 6].sum():.0f}, "
          f"advance {P[:, 14].sum() / P[:, 6].sum():.0f}), wait {P[:, 1].sum() / P[:, 6].sum():.0f}, math {P[:, 3].sum() / P[:, 6].sum():.0f}")
    h.close()
    t.close()
