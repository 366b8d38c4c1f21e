"""Accuracy of the product path against the fp64 oracle on every BASELINE config
(reading R16's statistics, tests/_tol.py): GPU tree + device ingest + P2P as
bench.py runs them, the oracle on all target leaves (C1, C2 at S = 32 / 128 / 512,
C5's snapshot) or on a seeded sample of >= 4096 leaves (C3, C4, C6), whose rows
are exact.  Writes one JSON object (profiles/r2_accuracy.json).

  python tools/accuracy_report.py [out.json]"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_ipps_overmanpmm13_b200 as afmm  # noqa: E402
import synth  # noqa: E402
from tests import _tol  # noqa: E402

oracle.build()
oracle.set_threads(len(os.sched_getaffinity(0)))
dev = torch.device("cuda", 0)
STREAM = torch.cuda.Stream(dev)        # one non-default stream shared by torch and both library handles
torch.cuda.set_stream(STREAM)


def gpu_eval(x, y, z, m, S, eps2, domain=None):
    # the tree, the P2P handle and torch share one stream: every read is ordered after its producer
    sp = STREAM.cuda_stream
    X, Y, Z, M = (torch.from_numpy(np.ascontiguousarray(v, np.float32)).to(dev) for v in (x, y, z, m))
    t = afmm.GpuTree(0, stream=sp)
    info = t.build(X, Y, Z, S, domain=domain)
    T = t.copy_out(x.shape[0])
    d = t.device_arrays()
    b = torch.empty((4, x.shape[0]), device=dev)
    for a, s in enumerate((X, Y, Z, M)):
        t.gather(s, b[a])
    h = afmm.P2P(eps2=eps2, stream=sp)
    h.set_bodies(b[0], b[1], b[2], b[3])
    h.set_tree_device(info["n_leaves"], d["leaf_start"], d["leaf_count"], d["u_off"], d["u_idx"])
    out = torch.empty((4, x.shape[0]), device=dev)
    h.eval(out[0], out[1], out[2], out[3])
    torch.cuda.synchronize()
    ax, ay, az, phi = out.cpu().numpy()
    h.close()
    t.close()
    return T, [phi, ax, ay, az]


def report(name, x, y, z, m, S, eps2, sample=None, domain=None, seed=0):
    t0 = time.time()
    T, got = gpu_eval(x, y, z, m, S, eps2, domain)
    To = oracle.Tree(x, y, z, S, domain=domain)
    for k in ("perm", "leaf_start", "leaf_count", "u_off", "u_idx"):
        assert np.array_equal(T[k], getattr(To, k)), (name, k)
    xs, ys, zs, ms = To.sorted_bodies(x, y, z, m)
    tg = None
    if sample:
        rng = np.random.default_rng(seed)
        tg = np.unique(np.concatenate([rng.choice(To.L, size=min(sample, To.L), replace=False),
                                       [0, To.L - 1, int(np.argmax(To.leaf_count))]])).astype(np.int32)
    ref = oracle.p2p(xs, ys, zs, ms, To.leaf_start, To.leaf_count, To.u_off, To.u_idx, 1.0, eps2, targets=tg,
                     with_scale=True)
    sel = np.ones(xs.shape[0], bool)
    if tg is not None:
        sel[:] = False
        for t in tg:
            sel[To.leaf_start[t]:To.leaf_start[t] + To.leaf_count[t]] = True
    st = _tol.check([g[sel] for g in got], [r[sel] for r in ref[:4]], ref[4][sel])
    st.update({"n": int(x.shape[0]), "S": S, "eps2": eps2, "bodies_checked": int(sel.sum()),
               "leaves_checked": int(To.L if tg is None else tg.size), "tree_bit_exact": True,
               "seconds": round(time.time() - t0, 1)})
    print(name, st, flush=True)
    return st


res = {"tolerance": {"rel": _tol.REL, "kappa": _tol.KAPPA, "abs_over_A_ill": _tol.ABS_A},
       "note": "phi per body relative; a global relative, per body relative where kappa <= 10, |da| <= 1e-6 A "
               "otherwise (reading R16); a_max_rel_all = the strict per-body max over every body"}
x, y, z, m = synth.make("C1")
res["C1"] = report("C1", x, y, z, m, 64, 1e-6)
x, y, z, m = synth.make("C2")
for S in (32, 128, 512):
    res[f"C2_S{S}"] = report(f"C2 S={S}", x, y, z, m, S, 1e-6)
x, y, z, m = synth.make("C3")
res["C3_sampled"] = report("C3", x, y, z, m, 128, 1e-6, sample=4096, seed=3)
x, y, z, m = synth.make("C4")
res["C4_sampled"] = report("C4", x, y, z, m, 256, 1e-6, sample=4096, seed=4)
x, y, z, m, vx, vy, vz = synth.colliding_with_velocities(1 << 20, 5)
res["C5_snapshot"] = report("C5", x, y, z, m, 128, 1e-4, domain=synth.c5_domain(x, y, z))
out = sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "profiles", "r2_accuracy.json")
json.dump(res, open(out, "w"), indent=1)
print("wrote", out)
