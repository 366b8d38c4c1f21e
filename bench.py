#!/usr/bin/env python
"""Benchmark of the AFMM near-field P2P hot path on B200 (BASELINE.json metric:
"near-field P2P interactions/s (and % FP32 peak) at 1/2/4/8 B200").

Workload (default): C4 = BASELINE configs[3], a 16M-body Plummer sphere at
leaf capacity S = 256 -- the configuration both north_star targets name (>= 60 %
of the FP32 peak on 1 GPU, >= 85 % parallel efficiency at 8 GPUs), and the
largest one that fits one GPU, so N = 1 and N > 1 measure the same workload
(strong scaling).  C2 (configs[1], 1M Plummer) is kept as the S sweep
32..512; C3 / C6 are extra lines.

One step = one pass of the whole hot path over the workload with inputs
resident in HBM: body ingest (pack on rank 0) and the P2P evaluation.
  N = 1: pack + P2P kernel.
  N > 1: the library communicator (afmm_p2p_config.nccl_id): rank 0 packs each
         chunk right before its broadcast (afmm_p2p_set_bodies_deferred), the
         eval broadcasts the packed bodies in chunks on a communication stream
         WHILE the P2P kernel runs (each warp waits only for the chunks its task
         needs), the kernel stores every result into every rank's output array
         over CUDA-IPC peer windows (fused gather), and one in-stream 8-byte
         all-reduce of the kernel time (the GPU time of PAPER L20 SVII.A) marks
         completion -- the only collective not overlapped with the kernel.
The tree is built once, on the GPU, by the product builder (afmm_tree_build)
and ingested on the device (afmm_p2p_set_tree_device); the workload is static.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C4] [--S 256]
  torchrun --nproc-per-node N bench.py --gpus N ...       (N > 1)
  python bench.py --impl reference ...                    (the fp64 oracle, CPU)

Prints ONE JSON line on rank 0.  Timing: CUDA events around each step on the
library's stream (= torch's current stream), L2 flushed (256 MiB write)
between steps outside the events (the 256 MiB of C4 bodies exceed L2 anyway),
barrier + synchronize on both sides, max over ranks.  Interactions =
sum_t n_t sum_{s in U(t)} n_s (PAPER L16 SIII.C); 20 flops per interaction
(the all-pairs convention of [14], north_star).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import synth  # noqa: E402  (seeded input generator shared by both arms)

E2E_PIECES = 1             # output pieces of the pipelined host-to-host evaluation (staged mode only)
FLOPS_PER_INTERACTION = 20
METRIC = "near-field P2P interactions/s (and % FP32 peak) at 1/2/4/8 B200"
SWEEP_S = [32, 48, 64, 96, 128, 192, 256, 384, 512]
WORKLOAD_DESC = {
    "C1": "4,096 uniform bodies in unit cube, S=64 (BASELINE configs[0])",
    "C2": "1M-body Plummer sphere (a=1, r<=10), 1 B200 (BASELINE configs[1])",
    "C3": "4M-body two colliding Plummer spheres, S=128 (BASELINE configs[2])",
    "C4": "16M-body Plummer sphere (a=1, r<=10), S=256 (BASELINE configs[3]; north_star's 1-GPU and 8-GPU targets)",
    "C5": "1M-body colliding galaxies (BASELINE configs[4], static snapshot)",
}
L2_NOTE = "flushed between steps (256 MiB write outside the step events)"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C4", choices=sorted(synth.CONFIGS))
    ap.add_argument("--S", type=int, default=None, help="leaf capacity (default: the config's)")
    ap.add_argument("--no-sweep", action="store_true", help="skip the C2 S sweep and the extra lines (N=1)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-stokeslet", action="store_true", help="skip the C6 Stokeslet line (N=1)")
    ap.add_argument("--no-proxy", action="store_true", help="skip the strong-scaling proxy (N=1)")
    ap.add_argument("--cpu-seconds", type=float, default=12.0, help="oracle sample budget (all cores)")
    ap.add_argument("--cpu-seconds-1core", type=float, default=6.0, help="oracle sample budget (1 core)")
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help="gloo + AFMM_BENCH_SAME_DEVICE=1 exercises the N>1 flow on one GPU (testing only)")
    return ap.parse_args()


def config_dict(name, S, n, n_leaves, nnz, inter, world):
    """The workload description both arms print (identical keys and values)."""
    c = synth.CONFIGS[name]
    return {"workload": WORKLOAD_DESC.get(name, name), "name": name, "S": S, "n": n, "eps2": c["eps2"],
            "seed": c["seed"], "n_leaves": int(n_leaves), "u_nnz": int(nnz), "interactions_per_step": int(inter),
            "l2": L2_NOTE, "parallelism": f"leaf-partition x{world} (cost model, PAPER L16)"}


def peak_fp32_tflops(sm_mhz=1965.0):
    """FP32 roofline from the unit counts (B200_PROFILING.md: 148 SMs; 128 FP32
    lanes per SM, 2 flop per FFMA) at the max SM clock (MEASURED_PEAKS.json)."""
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            sm_mhz = float(json.load(f).get("sm_max_mhz", sm_mhz))
    except Exception:
        pass
    return 148 * 128 * 2 * sm_mhz * 1e6 / 1e12, sm_mhz


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.proc = None
        self.lines = []

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                 "-lms", "20"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for ln in self.proc.stdout:
            self.lines.append(ln.strip())

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            p = [v.strip() for v in ln.split(",")]
            if len(p) < 9:
                continue
            try:
                sm.append(float(p[1]))
                mx = float(p[2])
            except ValueError:
                continue
            for nm, v in zip(names, p[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "samples": 0}
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sm)}


# ------------------------------------------------------------------ oracle legs (CPU)

def _oracle_sample(xs, ys, zs, ms, T, eps2, budget_s, seed=0):
    """Time the oracle's naive P2P on a seeded sample of target leaves sized to
    about budget_s seconds of CPU work.  Returns (interactions/s, desc, cores,
    interactions, seconds)."""
    import oracle
    I = oracle.interactions(T.leaf_count, T.u_off, T.u_idx)
    rng = np.random.default_rng(seed)
    order = rng.permutation(T.L).astype(np.int32)
    # probe ~0.05% of the work to estimate the rate
    cum = np.cumsum(I[order])
    k = int(np.searchsorted(cum, max(cum[-1] * 0.0005, 1)) + 1)
    t0 = time.perf_counter()
    oracle.p2p(xs, ys, zs, ms, T.leaf_start, T.leaf_count, T.u_off, T.u_idx, 1.0, eps2,
               targets=np.sort(order[:k]))
    rate = cum[k - 1] / max(time.perf_counter() - t0, 1e-6)
    want = min(cum[-1], rate * budget_s)
    k = int(min(T.L, np.searchsorted(cum, want) + 1))
    tg = np.sort(order[:k])
    t0 = time.perf_counter()
    oracle.p2p(xs, ys, zs, ms, T.leaf_start, T.leaf_count, T.u_off, T.u_idx, 1.0, eps2, targets=tg)
    dt = time.perf_counter() - t0
    inter = int(I[tg].sum())
    desc = (f"{k} of {T.L} target leaves ({inter:.4g} of {int(I.sum()):.4g} interactions, "
            f"{100.0 * inter / I.sum():.2f}%), seeded random, fp64 oracle_p2p")
    return inter / dt, desc, inter, dt


def _oracle_tree(name, S):
    import oracle
    oracle.build()
    x, y, z, m = synth.make(name)
    T = oracle.Tree(x, y, z, S)
    xs, ys, zs, ms = T.sorted_bodies(x, y, z, m)
    return T, xs, ys, zs, ms


def cpu_baseline(name, S, eps2, budget_all, budget_one):
    """The oracle as it stands on this host: all cores, then 1 core."""
    import oracle
    T, xs, ys, zs, ms = _oracle_tree(name, S)
    cores = len(os.sched_getaffinity(0))
    oracle.set_threads(cores)
    r_all, desc_all, _, _ = _oracle_sample(xs, ys, zs, ms, T, eps2, budget_all, seed=0)
    oracle.set_threads(1)
    r_one, desc_one, _, _ = _oracle_sample(xs, ys, zs, ms, T, eps2, budget_one, seed=1)
    oracle.set_threads(cores)
    return {"value": r_all, "unit": "interactions/s", "cores": cores, "kind": "oracle",
            "sample": f"{desc_all}, OpenMP {cores} threads",
            "one_core": {"value": r_one, "unit": "interactions/s", "cores": 1,
                         "sample": f"{desc_one}, 1 thread"}}


def run_reference(args):
    """--impl reference: the fp64 CPU oracle (the tier's reference arm) on the
    same workload, each step a bounded sample; rank 0 only."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import oracle
    c = synth.CONFIGS[args.config]
    S = args.S or c["S"]
    T, xs, ys, zs, ms = _oracle_tree(args.config, S)
    cores = len(os.sched_getaffinity(0))
    oracle.set_threads(cores)
    I = oracle.interactions(T.leaf_count, T.u_off, T.u_idx)
    steps, warm = max(1, args.steps), max(0, args.warmup)
    per_step = max(0.5, 150.0 / (steps + warm))
    total_i, total_t = 0, 0.0
    desc = None
    for i in range(steps + warm):
        r, desc, inter, dt = _oracle_sample(xs, ys, zs, ms, T, c["eps2"], per_step, seed=i)
        if i >= warm:
            total_i += inter
            total_t += dt
    value = total_i / total_t
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": "interactions/s",
            "n_gpus": args.gpus, "steps": steps, "warmup": warm,
            "ms_per_step": 1e3 * total_t / steps, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": config_dict(args.config, S, int(xs.shape[0]), T.L, int(T.u_off[-1]), int(I.sum()), args.gpus),
            "cpu_baseline": {"value": value, "unit": "interactions/s", "cores": cores, "kind": "oracle",
                             "sample": f"per step: {desc}, OpenMP {cores} threads"},
            "e2e": {"value": value, "unit": "interactions/s", "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------ our arm

def _gpu_tree(afmm, dev, stream, X, Y, Z, S):
    tree = afmm.GpuTree(dev.index, stream=stream.cuda_stream)
    t0 = time.perf_counter()
    info = tree.build(X, Y, Z, S)
    return tree, info, time.perf_counter() - t0


def extras_n1(args, afmm, torch, dev, stream, peak, kern_mean_main, main_dev_tree):
    """N = 1 extra lines: the C2 S sweep (and C2 S = 128, round 1's anchor), C3,
    the kernel-only strong-scaling proxy on the main workload, the Stokeslet C6."""
    extra = {}
    if not args.no_sweep:
        c2 = synth.CONFIGS["C2"]
        x, y, z, m = synth.make("C2")
        n = x.shape[0]
        X, Y, Z, M = (torch.from_numpy(v).to(dev) for v in (x, y, z, m))
        out = torch.empty((4, n), device=dev)
        sweep = {}
        for s2 in SWEEP_S:
            tr2, inf2, _ = _gpu_tree(afmm, dev, stream, X, Y, Z, s2)
            d2 = tr2.device_arrays()
            b2 = torch.empty((4, n), device=dev)
            for a, src in enumerate((X, Y, Z, M)):
                tr2.gather(src, b2[a])
            h2 = afmm.P2P(device=dev.index, eps2=c2["eps2"], stream=stream.cuda_stream)
            h2.set_bodies(b2[0], b2[1], b2[2], b2[3])
            h2.set_tree_device(inf2["n_leaves"], d2["leaf_start"], d2["leaf_count"], d2["u_off"], d2["u_idx"])
            for _ in range(8):
                h2.eval(out[0], out[1], out[2], out[3])
            km = float(np.median(h2.kernel_times(5)))
            s2st = h2.stats()
            ips = s2st["interactions_total"] / (km * 1e-3)
            sweep[str(s2)] = {"n_leaves": inf2["n_leaves"], "interactions": s2st["interactions_total"],
                              "kernel_ms": round(km, 4), "interactions_per_s": ips,
                              "frac_fp32": FLOPS_PER_INTERACTION * ips / (peak * 1e12)}
            if s2 == 128:
                # host tree ingest (afmm_p2p_set_tree: host arrays -> device ingest), C2 S=128
                T2 = tr2.copy_out(n)
                ts = []
                for _ in range(3):
                    t0 = time.perf_counter()
                    h2.set_tree(T2["leaf_start"], T2["leaf_count"], T2["u_off"], T2["u_idx"])
                    ts.append(time.perf_counter() - t0)
                extra["c2_host_set_tree_ms"] = round(1e3 * min(ts), 3)
            h2.close()
            tr2.close()
        extra["sweep_S"] = sweep
        extra["c2_s128"] = dict(sweep["128"], workload=WORKLOAD_DESC["C2"] + ", S=128 (round-1 headline)")
        del X, Y, Z, M, out
        # C3: two colliding Plummer spheres, 4M bodies, S = 128
        c3 = synth.CONFIGS["C3"]
        x, y, z, m = synth.make("C3")
        n3 = x.shape[0]
        X, Y, Z, M = (torch.from_numpy(v).to(dev) for v in (x, y, z, m))
        tr3, inf3, _ = _gpu_tree(afmm, dev, stream, X, Y, Z, c3["S"])
        d3 = tr3.device_arrays()
        b3 = torch.empty((4, n3), device=dev)
        for a, src in enumerate((X, Y, Z, M)):
            tr3.gather(src, b3[a])
        h3 = afmm.P2P(device=dev.index, eps2=c3["eps2"], stream=stream.cuda_stream)
        h3.set_bodies(b3[0], b3[1], b3[2], b3[3])
        h3.set_tree_device(inf3["n_leaves"], d3["leaf_start"], d3["leaf_count"], d3["u_off"], d3["u_idx"])
        o3 = torch.empty((4, n3), device=dev)
        for _ in range(6):
            h3.eval(o3[0], o3[1], o3[2], o3[3])
        k3 = float(np.median(h3.kernel_times(4)))
        i3 = h3.stats()["interactions_total"]
        extra["c3"] = {"workload": WORKLOAD_DESC["C3"], "interactions": i3, "kernel_ms": round(k3, 4),
                       "interactions_per_s": i3 / (k3 * 1e-3),
                       "frac_fp32": FLOPS_PER_INTERACTION * i3 / (k3 * 1e-3) / (peak * 1e12)}
        h3.close()
        tr3.close()
        del X, Y, Z, M, b3, o3

    if not args.no_proxy:
        # strong-scaling proxy of the kernel: every rank's work is independent (disjoint
        # target leaves, replicated sources), so rank r of a world-W partition is timed
        # alone on this GPU (one rebalance from the measured times)
        bod, info, d, n = main_dev_tree
        out = torch.empty((4, n), device=dev)
        proxy = {}
        for W in (2, 4, 8):
            hs = []
            for r in range(W):
                hw = afmm.P2P(device=dev.index, rank=r, world=W, eps2=synth.CONFIGS[args.config]["eps2"],
                              stream=stream.cuda_stream)
                hw.set_bodies(bod[0], bod[1], bod[2], bod[3])
                hw.set_tree_device(info["n_leaves"], d["leaf_start"], d["leaf_count"], d["u_off"], d["u_idx"])
                hs.append(hw)
            for it in range(2):
                ts = []
                for hw in hs:
                    for _ in range(4):
                        hw.eval(out[0], out[1], out[2], out[3])
                    ts.append(float(np.median(hw.kernel_times(3))))
                if it == 0:
                    for hw in hs:
                        hw.rebalance(np.array(ts), 0.02)
            proxy[str(W)] = {"rank_kernel_ms_max": round(max(ts), 4),
                             "E": round(kern_mean_main / (W * max(ts)), 3)}
            for hw in hs:
                hw.close()
        extra["strong_scaling_proxy"] = {
            "method": "kernel only: rank r of a world-W cost-model partition timed alone on one GPU after one "
                      "rebalance; E = T1 / (W * max_r T_r); no broadcast / gather / launch costs",
            "T1_ms": round(kern_mean_main, 4), "worlds": proxy}

    if not args.no_sweep:
        # row f1: the C5 dynamic workload (BASELINE configs[4]: 1M colliding bodies, leapfrog KDK with Enforce_S tree
        # maintenance and device ingest every step; fixed S = 128), 60 steps after 5 warm-up steps, one GPU
        from paper_conf_ipps_overmanpmm13_b200.timeloop import TimeLoop
        c5 = synth.CONFIGS["C5"]
        x5, y5, z5, m5, vx5, vy5, vz5 = synth.colliding_with_velocities(c5["n"], c5["seed"])
        loop = TimeLoop(x5, y5, z5, m5, vx5, vy5, vz5, c5["S"], c5["eps2"], 0.05, synth.c5_domain(x5, y5, z5),
                        device=dev.index)
        for _ in range(5):
            loop.step()
        # 60 steps back to back (no synchronise between steps: the next step's host work overlaps this
        # step's P2P kernel), one synchronise at the end; per-step phases from CUDA events
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        recs = [loop.step(sync=False) for _ in range(60)]
        loop.finish(recs)
        wall_ms = 1e3 * (time.perf_counter() - t0) / len(recs)
        keys = ("kernel_ms", "eval_ms", "enforce_ms", "set_tree_ms", "kick_drift_ms", "gpu_step_ms")
        mean = {k: round(float(np.mean([r[k] for r in recs])), 4) for k in keys}
        mean["step_ms"] = round(wall_ms, 4)
        inter = float(np.mean([r["interactions"] for r in recs]))
        extra["c5"] = {"workload": "C5: 1M colliding bodies, KDK dt=0.05, Enforce_S + device ingest every step, S=128, "
                                   "eps2=1e-4, 60 timed steps (BASELINE configs[4], one GPU)",
                       "mean_ms": mean, "interactions_per_step": inter,
                       "kernel_interactions_per_s": inter / (mean["kernel_ms"] * 1e-3),
                       "step_interactions_per_s": inter / (mean["step_ms"] * 1e-3),
                       "note": "step_ms = host wall time of 60 steps / 60 (steps enqueued back to back, one "
                               "synchronise at the end; every step still waits for its tree and work-list "
                               "readbacks); gpu_step_ms = CUDA-event span of one step"}
        loop.close()
        torch.cuda.set_stream(stream)

    if not args.no_stokeslet:
        # row f4: the regularized-Stokeslet law on its paper workload (C6: 10M uniform sources, L26 SIX.B)
        c6 = synth.CONFIGS["C6"]
        sx, sy, sz, sfx, sfy, sfz = synth.uniform_with_forces(c6["n"], c6["seed"])
        n6 = sx.shape[0]
        D = [torch.from_numpy(v).to(dev) for v in (sx, sy, sz, sfx, sfy, sfz)]
        tr6, inf6, _ = _gpu_tree(afmm, dev, stream, D[0], D[1], D[2], c6["S"])
        d6 = tr6.device_arrays()
        B6 = torch.empty((6, n6), device=dev)
        for a in range(6):
            tr6.gather(D[a], B6[a])
        h6 = afmm.P2P(device=dev.index, eps2=c6["eps2"], stream=stream.cuda_stream, law=afmm.LAW_STOKESLET)
        h6.set_bodies_stokeslet(*[B6[a] for a in range(6)])
        h6.set_tree_device(inf6["n_leaves"], d6["leaf_start"], d6["leaf_count"], d6["u_off"], d6["u_idx"])
        o6 = torch.empty((4, n6), device=dev)
        for _ in range(6):
            h6.eval(o6[0], o6[1], o6[2], o6[3])
        k6 = float(np.median(h6.kernel_times(4)))
        st6 = h6.stats()
        ips6 = st6["interactions_total"] / (k6 * 1e-3)
        extra["stokeslet_C6"] = {
            "workload": "C6: 10M uniform Stokeslet sources, S=128, eps2=1e-6 (PAPER L26 SIX.B; reading R26)",
            "interactions": st6["interactions_total"], "kernel_ms": k6, "interactions_per_s": ips6,
            "flop_per_interaction": 32, "frac_fp32": 32 * ips6 / (peak * 1e12),
            "note": "19 packed FP32 ops + 2 MUFU per two interactions; FMA=2 flop, rsqrt=1"}
        h6.close()
        tr6.close()
    return extra


def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)

    import torch
    import torch.distributed as dist
    import paper_conf_ipps_overmanpmm13_b200 as afmm
    from paper_conf_ipps_overmanpmm13_b200 import dist as pdist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if os.environ.get("AFMM_BENCH_SAME_DEVICE") == "1":     # functional test of the N>1 flow on one GPU
        local = 0
    torch.cuda.set_device(local)
    if world > 1:
        if args.dist_backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group("gloo")
    dev = torch.device("cuda", local)
    # a dedicated (non-default) stream shared by torch and the library, so the
    # step events and the library's work are ordered on one stream
    stream = torch.cuda.Stream(dev)
    torch.cuda.set_stream(stream)

    # FP32 FMA peak of this GPU, measured live (north_star "measured FP32 FMA peak")
    fp32 = afmm.fp32_peak(local) if rank == 0 else None
    peak, sm_max = peak_fp32_tflops()

    c = synth.CONFIGS[args.config]
    S = args.S or c["S"]
    eps2 = c["eps2"]
    x, y, z, m = synth.make(args.config)
    n = int(x.shape[0])

    # ---- setup (untimed): product GPU tree, bodies into tree order on device, device ingest
    X, Y, Z, M = (torch.from_numpy(v).to(dev) for v in (x, y, z, m))
    del x, y, z, m
    tree, info, tree_s = _gpu_tree(afmm, dev, stream, X, Y, Z, S)
    d = tree.device_arrays()
    bod = torch.empty((4, n), device=dev)
    for a, src in enumerate((X, Y, Z, M)):
        tree.gather(src, bod[a])
    del X, Y, Z, M
    torch.cuda.synchronize()

    # N > 1: the library communicator (chunked broadcast overlapped with the kernel,
    # in-stream GPU-time all-reduce); if it cannot be created, the caller-side path
    comm_mode = None
    h = None
    if world > 1 and args.dist_backend == "nccl":
        try:
            ids = [afmm.nccl_id() if rank == 0 else None]
            dist.broadcast_object_list(ids, src=0)
            h = afmm.P2P(device=local, rank=rank, world=world, G=1.0, eps2=eps2, stream=stream.cuda_stream,
                         nccl_id=ids[0])
            comm_mode = "library"
        except Exception as e:  # noqa: BLE001
            comm_mode = f"caller (library communicator unavailable: {e})"[:200]
            h = None
    if h is None:
        h = afmm.P2P(device=local, rank=rank, world=world, G=1.0, eps2=eps2, stream=stream.cuda_stream)
    if world == 1 or rank == 0:
        h.set_bodies(bod[0], bod[1], bod[2], bod[3])
    else:
        h.set_bodies(None, None, None, None, n=n)
    t0 = time.perf_counter()
    h.set_tree_device(info["n_leaves"], d["leaf_start"], d["leaf_count"], d["u_off"], d["u_idx"])
    set_tree_s = time.perf_counter() - t0
    out = torch.empty((4, n), device=dev)           # ax, ay, az, phi
    flush = torch.empty(64 << 20, dtype=torch.float32, device=dev)   # 256 MiB > 126 MB L2

    close_windows = None
    gather_mode = "none (N = 1)"
    if world > 1:
        # a7 fused: every rank's output array is a peer window of every other rank's
        # handle (CUDA IPC over NVLink); the P2P kernel stores each result into all of
        # them as its tasks finish.  If IPC is refused: NCCL allgatherv of the slices.
        try:
            close_windows = pdist.open_peer_windows(h, out)
            gather_mode = "fused: P2P kernel stores into CUDA-IPC peer windows"
        except Exception as e:  # noqa: BLE001
            gather_mode = f"NCCL allgatherv (peer windows unavailable: {e})"[:200]
    done = torch.zeros(1, device=dev)
    packed = pdist.packed_bodies(h, dev) if world > 1 and comm_mode != "library" else None

    def step():
        if world > 1 and rank == 0 and comm_mode == "library":
            h.set_bodies_deferred(bod[0], bod[1], bod[2], bod[3])   # a1: packed chunk by chunk inside the eval
        elif world == 1 or rank == 0:
            h.set_bodies(bod[0], bod[1], bod[2], bod[3])      # a1: pack (1 kernel; the root only at N > 1)
        elif comm_mode == "library":
            h.set_bodies(None, None, None, None, n=n)         # a4: to be received in the next eval
        if world > 1 and comm_mode != "library":
            dist.broadcast(packed, src=0)                     # a4 (caller path): ONE broadcast, not overlapped
        h.eval(out[0], out[1], out[2], out[3])                # a5/a6 (+ a4 chunked, a7 fused, a8 all-reduce)
        if world > 1 and close_windows is None:
            pdist.gather_slices([out[a] for a in range(4)], h.get_partition()[1])
        elif world > 1 and comm_mode != "library":            # caller path: completion of the peer stores
            if args.dist_backend == "nccl":
                dist.all_reduce(done)
            else:
                torch.cuda.synchronize()
                dist.barrier()

    # clocks are sampled from the warm-up through the timed region
    clk = ClockSampler(local).__enter__()

    # ---- warm-up (+ incremental rebalance from measured kernel times, L18 SIV.D)
    rebalanced = 0
    W_ = max(3, args.warmup)
    for i in range(W_):
        step()
        if world > 1:
            times = pdist.allgather_scalar(h.kernel_times(1)[-1], dev)
            if h.rebalance(times, 0.02):
                rebalanced += 1
    torch.cuda.synchronize()

    # ---- timed region
    K = args.steps
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    launches0 = afmm.launch_count()
    for k in range(K):
        flush.zero_()                                         # L2 flush, outside the step events
        ev[k][0].record(stream)
        step()
        ev[k][1].record(stream)
    torch.cuda.synchronize()
    launches = afmm.launch_count() - launches0
    clk.__exit__(None, None, None)
    if world > 1:
        dist.barrier()
    step_ms = [a.elapsed_time(b) for a, b in ev]
    kern_ms = h.kernel_times(K)
    st = h.stats()
    tot = torch.tensor([sum(step_ms), float(np.mean(kern_ms)), float(launches)], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(tot, op=dist.ReduceOp.MAX)
        lsum = torch.tensor([float(launches)], dtype=torch.float64, device=dev)
        dist.all_reduce(lsum)
        launches_all = int(lsum.item())
    else:
        launches_all = launches
    total_ms, kern_max = float(tot[0]), float(tot[1])
    inter = st["interactions_total"]
    value = inter * K / (total_ms * 1e-3)

    # ---- end to end through the public API with host buffers (H2D + D2H in the timed region)
    hx = [torch.empty(n, dtype=torch.float32).pin_memory() for _ in range(4)]
    for a in range(4):
        hx[a].copy_(bod[a].cpu())
    ho = [torch.empty(n, dtype=torch.float32).pin_memory() for _ in range(4)]
    Ke = max(3, K // 2)
    e2e_mode = {"zero_copy": 0, "input_graph": 0, "streamed_inputs": 0}

    def step_e2e():
        if world == 1:
            # afmm_p2p_eval_host_pipelined: inputs packed from the pinned host arrays while the
            # kernel runs, outputs written to the pinned host arrays by the task epilogue; blocking
            st_ = h.eval_host_pipelined(*hx, *ho, pieces=E2E_PIECES)
            for k_ in e2e_mode:
                e2e_mode[k_] = st_[k_]
        else:
            if rank == 0:
                for a in range(4):
                    bod[a].copy_(hx[a], non_blocking=True)
            step()
            if rank == 0:
                for a in range(4):
                    ho[a].copy_(out[a], non_blocking=True)
            torch.cuda.synchronize()

    step_e2e()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    # three blocks of Ke host-to-host steps (PCIe / host-memory hiccups move single blocks by a few %):
    # the median block's rate is the line's e2e, every block is reported
    blocks = []
    for _ in range(3):
        if world > 1:
            dist.barrier()
        t0 = time.perf_counter()
        for _ in range(Ke):
            step_e2e()
        torch.cuda.synchronize()
        e2e_s = torch.tensor([time.perf_counter() - t0], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(e2e_s, op=dist.ReduceOp.MAX)
        blocks.append(inter * Ke / float(e2e_s[0]))
    e2e_value = float(np.median(blocks))

    # ---- roofline of the dominant kernel (the P2P kernel): FP32 ALU bound
    kern_mean = float(np.mean(kern_ms))
    achieved = FLOPS_PER_INTERACTION * st["interactions_rank"] / (kern_mean * 1e-3) / 1e12
    prof_traffic = None
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
            tr = json.load(f)
            if tr.get("config") == args.config and tr.get("S") == S:
                prof_traffic = tr.get("dram_bytes_per_launch")
    except Exception:
        pass

    extra = {}
    if rank == 0 and world == 1:
        extra = extras_n1(args, afmm, torch, dev, stream, peak, kern_mean, (bod, info, d, n))

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        try:
            cpu = cpu_baseline(args.config, S, eps2, args.cpu_seconds, args.cpu_seconds_1core)
        except Exception as e:  # noqa: BLE001
            cpu = {"value": None, "unit": "interactions/s", "cores": None, "kind": "oracle",
                   "sample": f"failed: {e}"}

    if rank == 0:
        ffma = fp32["ffma_tflops"] if fp32 else None
        line = {
            "metric": METRIC, "value": value, "unit": "interactions/s", "n_gpus": world,
            "steps": K, "warmup": W_, "ms_per_step": total_ms / K,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f32",
            "data": "synthetic",
            "config": config_dict(args.config, S, n, info["n_leaves"], info["nnz"], inter, world),
            "step": {
                "what": ("pack + P2P kernel" if world == 1 else
                         ("eval: rank 0 packs each chunk right before its NCCL broadcast, the broadcasts overlapped with the "
                          "P2P kernel (library communicator) and followed by a tail grid of it on the NCCL SMs, kernel stores every "
                          "result into all ranks' outputs "
                          "over CUDA-IPC peer windows (fused gather), 8-byte in-stream all-reduce of the kernel "
                          "time = completion" if comm_mode == "library" else
                          "rank 0 packs + one NCCL broadcast of the packed bodies + P2P kernel storing into peer "
                          "windows + 4-byte all_reduce")),
                "communicator": comm_mode, "gather": gather_mode,
                "masses": "equal (1/N, reading R19): detected at pack time, equal-mass pair loop (12 packed FP32 "
                          "ops per pair, G m applied once; reading R30)",
                "tree_build_s": round(tree_s, 4), "set_tree_device_s": round(set_tree_s, 4)},
            "kernel_ms": {"mean": kern_mean, "median": float(np.median(kern_ms)), "best": float(np.min(kern_ms)),
                          "max_over_ranks": kern_max,
                          "kernel_ms_max_device_timer": st["kernel_ms_max"] if comm_mode == "library" else None},
            "gpu_time_interactions_per_s": inter / (kern_max * 1e-3),
            "roofline": {"bound": "alu", "achieved": achieved, "peak": peak, "unit": "TFLOP/s",
                         "frac": achieved / peak, "traffic": prof_traffic,
                         "peak_note": (f"derived: 148 SM x 128 FP32 lanes x 2 flop x {sm_max:.0f} MHz "
                                       "(guide's unit counts at MEASURED_PEAKS sm_max_mhz; no FP32 entry there); "
                                       "20 flop/interaction"),
                         "peak_measured": ffma, "frac_measured": (achieved / ffma) if ffma else None,
                         "peak_measured_note": "afmm_fp32_peak on this GPU in this run: FFMA, 4 CTAs x 256 threads "
                                               "per SM, 16 independent chains per thread",
                         "kernel": "afmm::p2p_kernel_t<Gravity>"},
            "fp32_measured": fp32,
            "clocks": clk.summary(),
            "e2e": {"value": e2e_value, "unit": "interactions/s", "blocks": [round(b, 1) for b in blocks],
                    "h2d_bytes_per_step": 16 * n,
                    "d2h_bytes_per_step": 16 * n, "steps": Ke,
                    "path": (("afmm_p2p_eval_host_pipelined, zero-copy: " + str(min(16, max(8, n >> 20))) +
                              " input chunks (" + ("quadratic" if n >= (8 << 20) else "equal") +
                              " boundaries) packed from the pinned host arrays over PCIe while the kernel runs" +
                              (" (the pack chain replayed from a captured CUDA graph)" if e2e_mode["input_graph"]
                               else "") +
                              ("" if e2e_mode["streamed_inputs"] else " [fallback: inputs packed before the launch]") +
                              ", outputs written to the pinned host arrays by the kernel's task epilogue")
                             if e2e_mode["zero_copy"] else
                             f"afmm_p2p_eval_host_pipelined (8 streamed input chunks, {E2E_PIECES} output pieces) "
                             "from pinned host arrays") if world == 1
                    else "rank 0 H2D + step + D2H"},
            "gpu_launches": launches_all,
            "gpu_launches_note": "this library's kernels in the timed region, all ranks (afmm_launch_count "
                                 "difference: pack + P2P per step, + the GPU-time kernel with the library "
                                 "communicator); NCCL's kernels not counted",
            "rebalanced_in_warmup": rebalanced,
            "cpu_baseline": cpu,
            "paper_context": "98x whole-AFMM speedup, 10 CPU cores + 4 Tesla C2050 vs 1 core, 1M Plummer (L24 SVIII.E)",
        }
        line.update(extra)
        print(json.dumps(line), flush=True)
    if close_windows is not None:
        close_windows()
    h.close()
    tree.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
