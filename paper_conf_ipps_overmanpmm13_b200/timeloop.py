"""C5 dynamic workload (BASELINE configs[4]): kick-drift-
kick leapfrog steps with Enforce_S tree maintenance and the incremental
partition rebalance, all through the C ABI (orchestration only -- every
arithmetic step runs in libafmm_p2p.so kernels).

Per time step (PAPER L16 SIII.D "the particle positions are updated ... and
then any tree optimizations are done to improve the run on the next time step";
L20 SVI.A Enforce_S; L18 SIV.D observational coefficients):
  1. kick(dt/2) with the current accelerations      (afmm_kick_drift: 1 and 2 in one kernel,
  2. drift(dt)                                         own slice; the same roundings as afmm_kick + afmm_drift)
  3. N > 1: replicate positions and velocities        (allgatherv of slices)
  4. Enforce_S on the moved bodies (fixed domain)     (afmm_tree_enforce)
  5. carry the state into the new tree order          (afmm_tree_gather)
  6. set_bodies / set_tree; N > 1: the cut uses the per-bucket cost
     coefficients fitted to the previous step's kernel times (afmm_cost_fit)
  7. near-field P2P                                    (afmm_p2p_eval)
  8. kick(dt/2) with the new accelerations

With a load balancer (lb=LoadBalancer(...)) step 4 follows
the controller's action from the previous step instead (PAPER L18 SV, L20-L22):
  KEEP     afmm_tree_rebuild(KEEP): the structure is kept, bodies re-binned
  REBUILD  afmm_tree_build with the new S (fixed domain)
  ENFORCE  afmm_tree_enforce(S), predict, and FineGrainedOptimize if the
           controller asks (afmm_fine_grained), predict again
  FINE     KEEP + afmm_fine_grained
and after step 7 the controller sees T_gpu = the measured P2P kernel time (max
over ranks) and T_cpu = sum_op C_op M(op), the far-field time MODELLED from the
operation counts of the tree (afmm_tree_farfield_counts; reading R29: the CPU
far field is out of scope, so its time is a model with per-op costs cpu_coef).

Note: the far field is out of scope (S10), so bodies move under the
near-field force only; C5 is a dynamic load for the GPU path, not a physical
simulation.
"""
from __future__ import annotations

import time

import numpy as np
import torch

from . import (LB_ENFORCE, LB_FINE, LB_KEEP, LB_REBUILD, TREE_KEEP, GpuTree, P2P, cost_fit, drift,
               kick, kick_drift, lb_predict)

# Default modelled far-field costs (seconds per operation: P2M, M2M, M2L, L2L,
# L2P), reading R29: translation operators of an order-p expansion cost
# O(p^4) flops and P2M / L2P O(p^2) per body; the default puts one M2L at 1 ns
# so that the modelled far field and the measured B200 near field cross near
# the S the bench sweep finds (not a measurement of any CPU).
CPU_COEF_DEFAULT = (0.5e-9, 1.0e-9, 1.0e-9, 1.0e-9, 0.5e-9)


class TimeLoop:
    def __init__(self, x, y, z, m, vx, vy, vz, S, eps2, dt, domain, device=0, rank=0, world=1, G=1.0,
                 lb=None, cpu_coef=CPU_COEF_DEFAULT, fine_group=0.05, fine_max_groups=16, slice_world=0):
        self.dev = torch.device("cuda", device)
        self.stream = torch.cuda.Stream(self.dev)
        torch.cuda.set_stream(self.stream)
        self.S, self.eps2, self.dt, self.rank, self.world = int(S), float(eps2), float(dt), rank, world
        self.n = int(x.shape[0])
        self.domain = domain
        self.lb = lb
        self.cpu_coef = np.asarray(cpu_coef, np.float64)
        self.fine_group, self.fine_max_groups = float(fine_group), int(fine_max_groups)
        self.next_action = LB_KEEP
        self.c_p2p = None                                       # s per interaction, observed (L18 SIV.D)
        n = self.n
        # state in tree order: rows x, y, z, m, vx, vy, vz
        src = torch.stack([torch.as_tensor(np.asarray(v, np.float32)) for v in (x, y, z, m, vx, vy, vz)]).to(self.dev)
        self.state = torch.empty((7, n), device=self.dev)
        self.tmp = torch.empty((7, n), device=self.dev)
        self.acc = torch.zeros((4, n), device=self.dev)        # ax, ay, az, phi
        self.tree = GpuTree(device, stream=self.stream.cuda_stream)
        self.tree.build(src[0], src[1], src[2], self.S, domain=domain)
        for a in range(7):
            self.tree.gather(src[a], self.state[a])
        # slice_world (afmm_p2p_config): the task slicing; equal slice_world gives bit-identical
        # accelerations -- hence trajectories -- at any world size and partition (DESIGN R17)
        self.h = P2P(device=device, rank=rank, world=world, G=G, eps2=eps2, stream=self.stream.cuda_stream,
                     slice_world=slice_world)
        self.step_no = 0
        self.log = []
        self._load_tree(host_copy=True)
        self._eval()

    # ------------------------------------------------------------------ pieces
    def _load_tree(self, host_copy=False):
        """Device-side ingest of the GPU tree (afmm_p2p_set_tree_device): no host
        round trip; a host copy of the tree is kept only for verification hooks."""
        info = self.tree.info()
        d = self.tree.device_arrays()
        s = self.state
        self.h.set_bodies(s[0], s[1], s[2], s[3])
        self.h.set_tree_device(info["n_leaves"], d["leaf_start"], d["leaf_count"], d["u_off"], d["u_idx"])
        self.T = self.tree.copy_out(self.n) if host_copy else info
        self.body_split = self.h.get_partition()[1]

    def _slice(self):
        lo, hi = int(self.body_split[self.rank]), int(self.body_split[self.rank + 1])
        return lo, hi

    def _eval(self):
        a = self.acc
        self.h.eval(a[0], a[1], a[2], a[3])

    def _kick(self):
        lo, hi = self._slice()
        s, a = self.state, self.acc
        kick(s[4, lo:hi], s[5, lo:hi], s[6, lo:hi], a[0, lo:hi], a[1, lo:hi], a[2, lo:hi], 0.5 * self.dt,
             self.stream.cuda_stream)

    def _drift(self):
        lo, hi = self._slice()
        s = self.state
        drift(s[0, lo:hi], s[1, lo:hi], s[2, lo:hi], s[4, lo:hi], s[5, lo:hi], s[6, lo:hi], self.dt,
              self.stream.cuda_stream)

    def _kick_drift(self):
        """kick(dt/2) then drift(dt) in one kernel (afmm_kick_drift: the same two roundings)."""
        lo, hi = self._slice()
        s, a = self.state, self.acc
        kick_drift(s[0, lo:hi], s[1, lo:hi], s[2, lo:hi], s[4, lo:hi], s[5, lo:hi], s[6, lo:hi], a[0, lo:hi],
                   a[1, lo:hi], a[2, lo:hi], 0.5 * self.dt, self.dt, self.stream.cuda_stream)

    def _refit(self):
        """N > 1: per-bucket coefficients from this step's kernel times (L18 SIV.D)."""
        if self.world == 1:
            return
        import torch.distributed as dist
        st = self.h.stats()
        mine = torch.tensor([st["kernel_ms"]] + [float(v) for v in st["bucket_interactions"]],
                            dtype=torch.float64, device=self.dev)
        allv = [torch.zeros_like(mine) for _ in range(self.world)]
        dist.all_gather(allv, mine)
        arr = np.stack([v.cpu().numpy() for v in allv])
        self.h.set_cost_coef(cost_fit(arr[:, 1:], arr[:, 0]))

    # ------------------------------------------------------------------ load balancing
    def _times(self):
        """(T_cpu modelled, T_gpu measured max over ranks, counts) of this step."""
        ms = float(self.h.stats()["kernel_ms"])
        if self.world > 1:
            import torch.distributed as dist
            t = torch.tensor([ms], dtype=torch.float64, device=self.dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ms = float(t.item())
        c = self.tree.farfield_counts()
        return lb_predict(c, self._coef6())[0], 1e-3 * ms, c

    def _coef6(self):
        return np.concatenate([self.cpu_coef, [self.c_p2p or 0.0]])

    def _predict(self):
        """The predicted compute time of the current tree (afmm_lb_predict, L18 SIV.D)."""
        return lb_predict(self.tree.farfield_counts(), self._coef6())[2]

    def _maintain(self, x, y, z):
        """Tree maintenance of this step (step 4): Enforce_S without a balancer,
        else the controller's pending action."""
        rec = {"action": None}
        if self.lb is None:
            self.tree.enforce(x, y, z, self.S)
            return rec
        a = self.next_action
        rec["action"] = ("keep", "rebuild", "enforce", "fine")[a]
        if a == LB_REBUILD:
            self.tree.build(x, y, z, self.S, domain=self.domain)
        elif a == LB_ENFORCE:
            self.tree.enforce(x, y, z, self.S)
            rec["t_pred"] = self._predict()
            if self.lb.predicted(rec["t_pred"]) == LB_FINE:
                r = self.tree.fine_grained(x, y, z, self.S, self._coef6(), 0, self.fine_group, self.fine_max_groups)
                rec["fine"] = r
                self.lb.predicted(r["t_after"])
        else:
            self.tree.rebuild(x, y, z, self.S, mode=TREE_KEEP)
            if a == LB_FINE:
                r = self.tree.fine_grained(x, y, z, self.S, self._coef6(), 0, self.fine_group, self.fine_max_groups)
                rec["fine"] = r
                self.lb.predicted(r["t_after"])
        return rec

    def _balance(self, rec):
        t_cpu, t_gpu, c = self._times()
        if c[5] > 0:
            self.c_p2p = t_gpu / float(c[5])
        a, S = self.lb.step(t_cpu, t_gpu)
        self.next_action, self.S = a, S
        st = self.lb.state()
        rec.update({"t_cpu_model": t_cpu, "t_gpu": t_gpu, "compute": max(t_cpu, t_gpu), "lb_state": st["state"],
                    "S_next": S, "next": ("keep", "rebuild", "enforce", "fine")[a]})

    # ------------------------------------------------------------------ one step
    def step(self, hooks=None, sync=True):
        """One KDK step.  hooks (optional dict of callables) receive the state
        for verification: 'pre_enforce'(x, y, z) with positions in the old tree
        order, 'post_maintain'(loop, rec) after the tree maintenance (loop.tree
        holds the new tree), 'post_eval'(loop) after the new accelerations.
        sync=False (no load balancer, no hooks): the step is only enqueued past
        the library's own readbacks -- no synchronise at its end, so the next
        step's host work overlaps this step's P2P kernel; the record's timings
        are filled in later by finish(records) after one synchronise."""
        if not sync and (self.lb is not None or hooks):
            raise ValueError("sync=False needs lb=None and no hooks")
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(6)]
        t0 = time.perf_counter()
        ev[0].record(self.stream)
        self._refit()
        self._kick_drift()
        if self.world > 1:
            from . import dist as pdist
            pdist.gather_slices([self.state[a] for a in (0, 1, 2, 4, 5, 6)], self.body_split)
        ev[1].record(self.stream)
        s = self.state
        if hooks and "pre_enforce" in hooks:
            torch.cuda.synchronize()
            hooks["pre_enforce"](s[0].cpu().numpy(), s[1].cpu().numpy(), s[2].cpu().numpy())
        lbrec = self._maintain(s[0], s[1], s[2])
        if hooks and "post_maintain" in hooks:
            hooks["post_maintain"](self, lbrec)
        self.tree.gather_rows(s, self.tmp)          # all 7 state rows into the new tree order, one kernel
        self.state, self.tmp = self.tmp, self.state
        ev[2].record(self.stream)
        self._load_tree(host_copy=bool(hooks))
        ev[3].record(self.stream)
        self._eval()
        ev[4].record(self.stream)
        self._kick()
        ev[5].record(self.stream)
        if not sync:
            rec = {"step": self.step_no, "n_leaves": self.T["n_leaves"], "interactions": self.h.interactions()[0],
                   "S": self.S, "_events": ev}
            self.log.append(rec)
            self.step_no += 1
            return rec
        torch.cuda.synchronize()
        st = self.h.stats()
        rec = {"step": self.step_no, "n_leaves": self.T["n_leaves"], "interactions": st["interactions_total"],
               "kernel_ms": st["kernel_ms"], "kick_drift_ms": ev[0].elapsed_time(ev[1]),
               "enforce_ms": ev[1].elapsed_time(ev[2]), "set_tree_ms": ev[2].elapsed_time(ev[3]),
               "eval_ms": ev[3].elapsed_time(ev[4]), "step_ms": 1e3 * (time.perf_counter() - t0),
               "leaf_split": self.h.get_partition()[0].tolist(), "S": self.S}
        if self.lb is not None:
            t1 = time.perf_counter()
            rec.update(lbrec)
            self._balance(rec)
            rec["lb_ms"] = 1e3 * (time.perf_counter() - t1)
        self.log.append(rec)
        self.step_no += 1
        if hooks and "post_eval" in hooks:
            hooks["post_eval"](self)
        return rec

    def finish(self, recs):
        """After steps taken with sync=False: synchronise once and fill each record's
        timings from its events and the library's kernel-time ring (last <= 64 evals)."""
        torch.cuda.synchronize()
        kt = self.h.kernel_times(len(recs)) if recs else []
        kt = list(kt)[-len(recs):] if recs else []
        for r, k in zip(recs, [None] * (len(recs) - len(kt)) + kt):
            ev = r.pop("_events")
            r.update({"kernel_ms": k, "kick_drift_ms": ev[0].elapsed_time(ev[1]),
                      "enforce_ms": ev[1].elapsed_time(ev[2]), "set_tree_ms": ev[2].elapsed_time(ev[3]),
                      "eval_ms": ev[3].elapsed_time(ev[4]), "gpu_step_ms": ev[0].elapsed_time(ev[5])})
        return recs

    def close(self):
        self.h.close()
        self.tree.close()
