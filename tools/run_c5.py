"""Run the C5 dynamic workload (BASELINE configs[4]) on one GPU and report
per-step timings as one JSON line:
  python tools/run_c5.py [--n 1048576] [--steps 200] [--S 128] [--check-every 50]
With --check-every k, the step's Enforce_S tree is compared bit-exactly with the
oracle chain and P2P on 256 sampled leaves against the oracle (test infra)."""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402

import synth  # noqa: E402
from paper_conf_ipps_overmanpmm13_b200.timeloop import TimeLoop  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--n", type=int, default=1 << 20)
ap.add_argument("--steps", type=int, default=200)
ap.add_argument("--S", type=int, default=128)
ap.add_argument("--dt", type=float, default=0.05)
ap.add_argument("--eps2", type=float, default=1e-4)
ap.add_argument("--check-every", type=int, default=0)
ap.add_argument("--lb", action="store_true", help="drive S and the tree with the load balancer (row f3)")
ap.add_argument("--cpu-coef", default="", help="modelled far-field costs P2M,M2M,M2L,L2L,L2P (s/op)")
ap.add_argument("--no-fine", action="store_true", help="load balancer without FineGrainedOptimize")
a = ap.parse_args()
x, y, z, m, vx, vy, vz = synth.colliding_with_velocities(a.n, 5)
dom = synth.c5_domain(x, y, z)
t0 = time.perf_counter()
kw = {}
if a.lb:
    import paper_conf_ipps_overmanpmm13_b200 as afmm
    kw["lb"] = afmm.LoadBalancer(S_init=a.S)
    if a.cpu_coef:
        kw["cpu_coef"] = [float(v) for v in a.cpu_coef.split(",")]
    if a.no_fine:
        kw["fine_max_groups"] = 0
loop = TimeLoop(x, y, z, m, vx, vy, vz, a.S, a.eps2, a.dt, dom, **kw)
setup_s = time.perf_counter() - t0
checks = []
otree = [None]
if a.check_every:
    import oracle
    from tests import _tol
    otree[0] = oracle.Tree(x, y, z, a.S, domain=dom)


def pre(px, py, pz):
    otree[0] = otree[0].enforce(px, py, pz)


def post(lp):
    if lp.step_no % a.check_every:
        return
    import oracle
    from tests import _tol
    To = otree[0]
    same = all(np.array_equal(lp.T[k], getattr(To, k)) for k in ("leaf_start", "leaf_count", "u_off", "u_idx"))
    s = lp.state.cpu().numpy()
    acc = lp.acc.cpu().numpy()
    rng = np.random.default_rng(lp.step_no)
    tg = np.sort(rng.choice(To.L, size=min(256, To.L), replace=False)).astype(np.int32)
    ref = oracle.p2p(s[0], s[1], s[2], s[3], To.leaf_start, To.leaf_count, To.u_off, To.u_idx, 1.0, a.eps2,
                     targets=tg, with_scale=True)
    sel = np.zeros(a.n, bool)
    for t in tg:
        sel[To.leaf_start[t]:To.leaf_start[t] + To.leaf_count[t]] = True
    err = _tol.check([acc[3][sel], acc[0][sel], acc[1][sel], acc[2][sel]], [r[sel] for r in ref[:4]], ref[4][sel])
    checks.append({"step": lp.step_no, "tree_bit_exact": bool(same), **err})


hooks = {"pre_enforce": pre, "post_eval": post} if a.check_every else None
t0 = time.perf_counter()
for _ in range(a.steps):
    loop.step(hooks)
wall = time.perf_counter() - t0
L = loop.log
tot_int = sum(r["interactions"] for r in L)
tot_kernel = sum(r["kernel_ms"] for r in L) * 1e-3
print(json.dumps({
    "workload": f"C5: {a.n} colliding bodies, {a.steps} KDK steps, dt={a.dt}, S={a.S}, eps2={a.eps2}, 1 GPU",
    "setup_s": round(setup_s, 3), "wall_s": round(wall, 3),
    "interactions_total": tot_int, "kernel_interactions_per_s": tot_int / tot_kernel,
    "step_interactions_per_s": tot_int / sum(r["step_ms"] * 1e-3 for r in L),
    "mean_ms": {k: float(np.mean([r[k] for r in L])) for k in
                ("kernel_ms", "kick_drift_ms", "enforce_ms", "set_tree_ms", "eval_ms", "step_ms")},
    "step_ms_by_quarter": [round(float(np.mean([r["step_ms"] for r in L[q * len(L) // 4:(q + 1) * len(L) // 4]])), 3)
                           for q in range(4)],
    "set_tree_ms_by_quarter": [round(float(np.mean([r["set_tree_ms"] for r in L[q * len(L) // 4:(q + 1) * len(L) // 4]])), 3)
                               for q in range(4)],
    "n_leaves": [L[0]["n_leaves"], L[len(L) // 2]["n_leaves"], L[-1]["n_leaves"]],
    "interactions_per_step": [L[0]["interactions"], L[len(L) // 2]["interactions"], L[-1]["interactions"]],
    "checks": checks,
    **({"lb": {"cpu_coef": list(map(float, loop.cpu_coef)),
               "trajectory": [{k: (round(v, 7) if isinstance(v, float) else v) for k, v in r.items()
                               if k in ("step", "S", "action", "lb_state", "t_cpu_model", "t_gpu", "compute",
                                        "n_leaves", "lb_ms", "step_ms", "enforce_ms")} for r in L],
               "fine": [dict(step=r["step"], **r["fine"]) for r in L if "fine" in r],
               "compute_ms_by_quarter": [round(1e3 * float(np.mean([r["compute"] for r in
                                                                    L[q * len(L) // 4:(q + 1) * len(L) // 4]])), 4)
                                         for q in range(4)]}} if a.lb else {})}))
loop.close()
