"""Multi-rank host logic on CPU: world size 2 over gloo (127.0.0.1).

Exercises the same plumbing bench.py uses on NCCL (replicate bodies, gather
disjoint output slices, all-gather kernel times), the library's host-only cost
model (Interactions, literal partition, rebalance) on every rank, and checks
that the gathered result equals the single-rank result bit-exactly.  The
per-rank P2P compute is the oracle here (CPU test infrastructure standing in
for the kernel, which needs a GPU)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    try:
        import sys
        sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
        import oracle
        import paper_conf_ipps_overmanpmm13_b200 as afmm
        from paper_conf_ipps_overmanpmm13_b200 import dist as pdist
        import synth
        dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
        x, y, z, m = synth.make("plummer", 6000, 12)
        T = oracle.Tree(x, y, z, 24)
        xs, ys, zs, ms = T.sorted_bodies(x, y, z, m)
        n = xs.shape[0]
        # a4: only rank 0 holds the bodies; replicate them
        bod = torch.zeros((4, n), dtype=torch.float32)
        if rank == 0:
            bod[:] = torch.from_numpy(np.stack([xs, ys, zs, ms]))
        pdist.replicate([bod[a] for a in range(4)], src=0)
        assert np.array_equal(bod.numpy(), np.stack([xs, ys, zs, ms]))
        # a2/a3: the cost model on every rank (identical inputs -> identical cut)
        I = afmm.interactions(T.leaf_count, T.u_off, T.u_idx)
        split = afmm.partition_literal(I, world)
        bsplit = pdist.body_split_from(split, T.leaf_start, n)
        # a5 stand-in: this rank's target leaves only
        mine = np.arange(split[rank], split[rank + 1], dtype=np.int32)
        ref = oracle.p2p(*bod.numpy(), T.leaf_start, T.leaf_count, T.u_off, T.u_idx, 1.0, 1e-6, targets=mine)
        out = torch.full((4, n), float("nan"), dtype=torch.float32)
        lo, hi = bsplit[rank], bsplit[rank + 1]
        for a in range(4):
            out[a, lo:hi] = torch.from_numpy(ref[a][lo:hi].astype(np.float32))
        # a7: gather every rank's slice to all ranks
        pdist.gather_slices([out[a] for a in range(4)], bsplit)
        full = oracle.p2p(xs, ys, zs, ms, T.leaf_start, T.leaf_count, T.u_off, T.u_idx, 1.0, 1e-6)
        for a in range(4):
            assert np.array_equal(out[a].numpy(), full[a].astype(np.float32))
        # a8: per-rank "kernel times" (rank 1 twice as slow per interaction), rebalance on both ranks
        my_ms = float(I[split[rank]:split[rank + 1]].sum()) * (1e-9 if rank == 0 else 2e-9)
        times = pdist.allgather_scalar(my_ms, "cpu")
        new, changed = afmm.partition_rebalance(T.leaf_count, I, split, times, 0.02)
        allnew = [torch.zeros(world + 1, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(allnew, torch.from_numpy(new))
        q.put((rank, "ok", changed, [a.tolist() for a in allnew], split.tolist()))
        dist.destroy_process_group()
    except Exception as e:  # noqa: BLE001
        import traceback
        q.put((rank, "err", traceback.format_exc(), None, None))


def test_gloo_world2_replicate_gather_partition_rebalance():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in ps:
        p.join(timeout=60)
    for r in res:
        assert r[1] == "ok", r[2]
    # both ranks adopted the same new cut, which moves leaves off the slow rank 1
    _, _, changed, allnew, split = res[0]
    assert changed and allnew[0] == allnew[1]
    assert allnew[0][1] > split[1]


def test_rebalance_rule_host_only():
    import oracle
    import paper_conf_ipps_overmanpmm13_b200 as afmm
    import synth
    x, y, z, m = synth.make("plummer", 20000, 3)
    T = oracle.Tree(x, y, z, 32)
    I = afmm.interactions(T.leaf_count, T.u_off, T.u_idx)
    split = afmm.partition_literal(I, 4)
    # balanced times -> no change
    new, ch = afmm.partition_rebalance(T.leaf_count, I, split, [1.0, 1.0, 1.0, 1.0], 0.02)
    assert not ch and np.array_equal(new, split)
    # rank 2 slow -> its range shrinks; cut stays a valid partition; deterministic
    new, ch = afmm.partition_rebalance(T.leaf_count, I, split, [1.0, 1.0, 1.6, 1.0], 0.02)
    new2, _ = afmm.partition_rebalance(T.leaf_count, I, split, [1.0, 1.0, 1.6, 1.0], 0.02)
    assert ch and np.array_equal(new, new2)
    assert new[0] == 0 and new[-1] == T.L and (np.diff(new) >= 0).all()
    assert (new[3] - new[2]) < (split[3] - split[2])
    with pytest.raises(afmm.AfmmError):
        afmm.partition_rebalance(T.leaf_count, I, split, [1.0, np.nan, 1.0, 1.0], 0.02)
