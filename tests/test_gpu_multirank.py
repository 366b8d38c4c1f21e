"""The N > 1 path end to end with real kernels on ONE GPU: two ranks (gloo
backend, both on cuda:0) replicate the bodies from rank 0, evaluate their own
target leaves, rebalance from measured kernel times and gather the output
slices (paper_conf_ipps_overmanpmm13_b200.dist, the same helpers bench.py uses
over NCCL).  The gathered result must equal the single-rank result bit-exactly
(the partition never changes a result, R17)."""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


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
        import torch.distributed as dist
        import paper_conf_ipps_overmanpmm13_b200 as afmm
        from paper_conf_ipps_overmanpmm13_b200 import dist as pdist
        import synth
        torch.cuda.set_device(0)
        dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
        dev = torch.device("cuda", 0)
        x, y, z, m = synth.make("plummer", 300000, 14)
        n = x.shape[0]
        X, Y, Z, M = (torch.from_numpy(v).to(dev) for v in (x, y, z, m))
        tree = afmm.GpuTree(0)
        tree.build(X, Y, Z, 64)
        T = tree.copy_out(n)
        bod = torch.zeros((4, n), device=dev)
        if rank == 0:
            for a, src in enumerate((X, Y, Z, M)):
                tree.gather(src, bod[a])
        torch.cuda.synchronize()
        pdist.replicate([bod[a] for a in range(4)], src=0)
        h = afmm.P2P(device=0, rank=rank, world=world, eps2=1e-6)
        h.set_bodies(bod[0], bod[1], bod[2], bod[3])
        h.set_tree(T["leaf_start"], T["leaf_count"], T["u_off"], T["u_idx"])
        results = []
        for it in range(2):
            out = torch.full((4, n), float("nan"), device=dev)
            h.eval(out[0], out[1], out[2], out[3])
            torch.cuda.synchronize()
            pdist.gather_slices([out[a] for a in range(4)], h.get_partition()[1])
            results.append(out.cpu().numpy())
            times = pdist.allgather_scalar(h.kernel_times(1)[-1] * (1.0 if rank == 0 else 1.5), dev)
            h.rebalance(times, 0.0)
        split = h.get_partition()[0]
        ref = None
        if rank == 0:
            h1 = afmm.P2P(device=0, eps2=1e-6, slice_world=world)   # the ranks' task slicing
            h1.set_bodies(bod[0], bod[1], bod[2], bod[3])
            h1.set_tree(T["leaf_start"], T["leaf_count"], T["u_off"], T["u_idx"])
            o1 = torch.empty((4, n), device=dev)
            h1.eval(o1[0], o1[1], o1[2], o1[3])
            torch.cuda.synchronize()
            ref = o1.cpu().numpy()
            h1.close()
        ok = all(np.isfinite(r).all() for r in results)
        same = ref is None or all(np.array_equal(r, ref) for r in results)
        q.put((rank, "ok", ok, same, split.tolist()))
        h.close()
        tree.close()
        dist.destroy_process_group()
    except Exception:  # noqa: BLE001
        import traceback
        q.put((rank, "err", traceback.format_exc(), None, None))


def test_two_ranks_one_gpu_bit_identical_to_single_rank():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = sorted([q.get(timeout=600) for _ in range(2)])
    for p in ps:
        p.join(timeout=120)
    for r in res:
        assert r[1] == "ok", r[2]
        assert r[2], "non-finite gathered output"
        assert r[3], "gathered output differs from the single-rank result"
    assert res[0][4] == res[1][4]          # both ranks agree on the (rebalanced) cut
