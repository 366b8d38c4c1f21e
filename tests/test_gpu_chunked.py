"""Chunked body replication overlapped with the P2P kernel (SURVEY S8(a) row a4,
S8(e); PAPER L16 SIII.C "building the data to send to the GPUs"), the library
communicator of afmm_p2p_config.nccl_id, the GPU-time all-reduce (row a8,
L20 SVII.A), and the streamed-input fallbacks of afmm_p2p_eval_host_pipelined.

Every check is bit-exact against afmm_p2p_eval on the same partition: a
target's sums depend only on its task (R17), not on when its
sources arrived or on the order tasks run in."""
import os
import socket

import numpy as np
import pytest

import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


def _afmm():
    import paper_conf_ipps_overmanpmm13_b200 as afmm
    return afmm


def _setup(n=120000, S=64, seed=31, unequal=False):
    afmm = _afmm()
    x, y, z, m = synth.make("plummer", n, seed)
    if unequal:
        m = (m * np.random.default_rng(seed).uniform(0.5, 1.5, n)).astype(np.float32)
    X, Y, Z, M = (torch.from_numpy(v).cuda() for v in (x, y, z, m))
    tree = afmm.GpuTree(0)
    tree.build(X, Y, Z, S)
    T = tree.copy_out(n)
    bod = torch.empty((4, n), device="cuda")
    for a, src in enumerate((X, Y, Z, M)):
        tree.gather(src, bod[a])
    torch.cuda.synchronize()
    tree.close()
    return bod, T


def _plain(bod, T, world=1, rank=0, slice_world=0):
    afmm = _afmm()
    n = bod.shape[1]
    out = torch.full((4, n), float("nan"), device="cuda")
    h = afmm.P2P(rank=rank, world=world, eps2=1e-6, slice_world=slice_world)
    h.set_bodies(bod[0], bod[1], bod[2], bod[3])
    h.set_tree(T["leaf_start"], T["leaf_count"], T["u_off"], T["u_idx"])
    h.eval(out[0], out[1], out[2], out[3])
    lo, hi = h.get_partition()[1][rank:rank + 2]
    torch.cuda.synchronize()
    h.close()
    return out.cpu().numpy(), int(lo), int(hi)


@pytest.mark.parametrize("unequal", [False, True])
def test_library_communicator_one_rank(unequal):
    """A 1-rank library communicator through the C ABI: the eval after
    set_bodies runs the chunked path (NCCL broadcast of the trailer + chunks on
    the communication stream, kernel waiting per task, then a tail grid of the same
    kernel on the communication SMs draining the same task queue), the next eval
    the plain one; both bit-identical to a handle without communicator;
    kernel_ms_max is the all-reduced device-timer span (one rank: its own)."""
    afmm = _afmm()
    bod, T = _setup(unequal=unequal)
    ref, _, _ = _plain(bod, T)
    n = bod.shape[1]
    h = afmm.P2P(eps2=1e-6, nccl_id=afmm.nccl_id(), stream=torch.cuda.current_stream().cuda_stream)
    h.set_bodies(bod[0], bod[1], bod[2], bod[3])
    h.set_tree(T["leaf_start"], T["leaf_count"], T["u_off"], T["u_idx"])
    for it in range(3):
        out = torch.full((4, n), float("nan"), device="cuda")
        st = h.eval(out[0], out[1], out[2], out[3], stats=True)
        assert st["chunked_bodies"] == (1 if it == 0 else 0)
        # the chunked eval also runs the tail grid on the communication SMs after the broadcast (2 launches)
        assert st["n_launches"] == (2 if it == 0 else 1), st
        assert 0.3 * st["kernel_ms"] <= st["kernel_ms_max"] <= 3.0 * st["kernel_ms"] + 0.05, st
        assert np.array_equal(out.cpu().numpy(), ref)
    K, order = h.chunks()[0].shape[0] - 1, h.chunks()[1]
    assert sorted(order.tolist()) == list(range(K))
    # the root's deferred pack: every chunk packed right before its broadcast, inside the eval
    h.set_bodies_deferred(bod[0], bod[1], bod[2], bod[3])
    out = torch.full((4, n), float("nan"), device="cuda")
    st = h.eval(out[0], out[1], out[2], out[3], stats=True)
    assert st["chunked_bodies"] == 1
    assert np.array_equal(out.cpu().numpy(), ref)
    # a deferred pack that afmm_p2p_bodies_buffer needs first is packed in full
    h.set_bodies_deferred(bod[0], bod[1], bod[2], bod[3])
    ptr, nbytes = h.bodies_buffer()
    assert nbytes == 16 * (n + 1)
    out.fill_(float("nan"))
    h.eval(out[0], out[1], out[2], out[3])
    torch.cuda.synchronize()
    assert np.array_equal(out.cpu().numpy(), ref)
    # host outputs (afmm_p2p_eval_host) through the same communicator, after a new set_bodies
    h.set_bodies(bod[0], bod[1], bod[2], bod[3])
    ho = [np.full(n, np.nan, np.float32) for _ in range(4)]
    st = h.eval(*ho)
    assert st["chunked_bodies"] == 1
    assert np.array_equal(np.stack(ho), ref)
    h.close()


def test_eval_chunked_caller_delivery_and_timeout():
    """afmm_p2p_eval_chunked + afmm_p2p_publish_chunks in one process: ranks of a
    world-3 partition, each handle allocated empty (set_bodies(None)), the kernel
    launched first, then the trailer and every chunk copied in delivery order
    from a root handle's packed array on a side stream, each published; every
    rank's slice bit-identical to afmm_p2p_eval.  Then an eval whose chunks never
    come: the bounded wait reports AFMM_ECUDA instead of hanging."""
    afmm = _afmm()
    bod, T = _setup(n=90000, S=48, seed=7)
    n = bod.shape[1]
    world = 3
    root = afmm.P2P(eps2=1e-6)
    root.set_bodies(bod[0], bod[1], bod[2], bod[3])
    rp, rbytes = root.bodies_buffer()
    from paper_conf_ipps_overmanpmm13_b200 import dist as pdist
    src = torch.as_tensor(pdist._DeviceArray(rp, rbytes), device="cuda")
    side = torch.cuda.Stream()
    for r in range(world):
        ref, lo, hi = _plain(bod, T, world=world, rank=r)
        h = afmm.P2P(rank=r, world=world, eps2=1e-6, stream=torch.cuda.current_stream().cuda_stream)
        h.set_bodies(None, None, None, None, n=n)
        h.set_tree(T["leaf_start"], T["leaf_count"], T["u_off"], T["u_idx"])
        bounds, order = h.chunks()
        assert bounds[0] == 0 and bounds[-1] == n and len(order) == len(bounds) - 1
        # rank r receives a chunk of its own slice among the first `world` deliveries
        own = [c for c in range(len(order)) if lo <= bounds[c] < hi]
        if own:
            assert min(order.tolist().index(c) for c in own) < world
        dp, dbytes = h.bodies_buffer()
        dst = torch.as_tensor(pdist._DeviceArray(dp, dbytes), device="cuda")
        out = torch.full((4, n), float("nan"), device="cuda")
        # the side stream must be ordered after the handle's earlier work BEFORE the
        # kernel is enqueued (waiting on the stream after it would wait for the kernel,
        # which waits for the chunks: the bounded wait would report a timeout)
        side.wait_stream(torch.cuda.current_stream())
        h.eval_chunked(out[0], out[1], out[2], out[3])
        with torch.cuda.stream(side):
            dst[4 * n:].copy_(src[4 * n:])                       # trailer (equal-mass flag, m_0)
            for j, c in enumerate(order):
                a, b = 4 * int(bounds[c]), 4 * int(bounds[c + 1])
                dst[a:b].copy_(src[a:b])
                h.publish_chunks(j + 1, side.cuda_stream)
        st = h.stats()
        assert st["chunked_bodies"] == 1
        got = out.cpu().numpy()
        assert np.array_equal(got[:, lo:hi], ref[:, lo:hi]), r
        h.close()
    # never delivered: bounded wait -> AFMM_ECUDA at the synchronising stats call
    h = afmm.P2P(eps2=1e-6)
    h.set_bodies(None, None, None, None, n=n)
    h.set_tree(T["leaf_start"], T["leaf_count"], T["u_off"], T["u_idx"])
    out = torch.empty((4, n), device="cuda")
    h.eval_chunked(out[0], out[1], out[2], out[3])
    with pytest.raises(afmm.AfmmError, match="never arrived"):
        h.stats()
    h.close()
    root.close()


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
        os.environ["AFMM_WAIT_MS"] = "60000"     # two processes time-slice one GPU
        import torch.distributed as dist
        import paper_conf_ipps_overmanpmm13_b200 as afmm
        from paper_conf_ipps_overmanpmm13_b200 import dist as pdist
        torch.cuda.set_device(0)
        dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
        bod, T = _setup(n=150000, S=64, seed=11)
        n = bod.shape[1]
        main = torch.cuda.current_stream()
        h = afmm.P2P(rank=rank, world=world, eps2=1e-6, stream=main.cuda_stream)
        if rank == 0:
            h.set_bodies(bod[0], bod[1], bod[2], bod[3])
        else:
            h.set_bodies(None, None, None, None, n=n)
        h.set_tree(T["leaf_start"], T["leaf_count"], T["u_off"], T["u_idx"])
        side = torch.cuda.Stream()
        results = []
        for it in range(2):
            out = torch.full((4, n), float("nan"), device="cuda")
            side.wait_stream(main)                               # earlier readers of the bodies
            h.eval_chunked(out[0], out[1], out[2], out[3])      # kernel first ...
            pdist.deliver_chunks(h, side, src=0)                 # ... bodies while it runs
            st = h.stats()
            torch.cuda.synchronize()
            pdist.gather_slices([out[a] for a in range(4)], h.get_partition()[1])
            results.append((out.cpu().numpy(), st["chunked_bodies"]))
        ref = None
        if rank == 0:
            ref, _, _ = _plain(bod, T, slice_world=world)         # the ranks' task slicing
        same = ref is None or all(np.array_equal(r, ref) for r, _ in results)
        q.put((rank, "ok", all(c == 1 for _, c in results), same))
        h.close()
        dist.destroy_process_group()
    except Exception:  # noqa: BLE001
        import traceback
        q.put((rank, "err", traceback.format_exc(), None))


@pytest.mark.parametrize("world", [2, 3])
def test_chunked_replication_gloo_ranks_one_gpu(world):
    """world processes on one GPU (gloo): rank 0 packs, every rank launches the
    chunk-waiting kernel, then the chunks are broadcast (dist.deliver_chunks) and
    published while it runs; the gathered result equals world = 1 bit for bit."""
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = sorted([q.get(timeout=600) for _ in range(world)])
    for p in ps:
        p.join(timeout=120)
    for r in res:
        assert r[1] == "ok", r[2]
        assert r[2], "an eval did not run the chunked path"
        assert r[3], "gathered output differs from the single-rank result"


def test_pipelined_rank_slice_inputs_change_between_calls():
    """afmm_p2p_eval_host_pipelined on a rank of world 2 must join its
    input chain before returning -- the second call (new host inputs) must not
    see the first call's chunk flags or bodies.  Each call equals
    afmm_p2p_eval on the same bodies, on the rank's slice."""
    afmm = _afmm()
    bod, T = _setup(n=100000, S=64, seed=5)
    n = bod.shape[1]
    bod2 = bod.clone()
    bod2[:3] += 1e-4 * torch.randn((3, n), device="cuda")        # same tree, moved bodies
    for r in range(2):
        h = afmm.P2P(rank=r, world=2, eps2=1e-6)
        h.set_bodies(bod[0], bod[1], bod[2], bod[3])
        h.set_tree(T["leaf_start"], T["leaf_count"], T["u_off"], T["u_idx"])
        lo, hi = (int(v) for v in h.get_partition()[1][r:r + 2])
        for b in (bod, bod2, bod, bod2):
            hb = [b[a].cpu().pin_memory() for a in range(4)]
            got = [torch.full((n,), float("nan")).pin_memory() for _ in range(4)]
            h.eval_host_pipelined(*hb, *got, pieces=1)
            ref = torch.full((4, n), float("nan"), device="cuda")
            hr = afmm.P2P(rank=r, world=2, eps2=1e-6)
            hr.set_bodies(b[0], b[1], b[2], b[3])
            hr.set_tree(T["leaf_start"], T["leaf_count"], T["u_off"], T["u_idx"])
            hr.eval(ref[0], ref[1], ref[2], ref[3])
            torch.cuda.synchronize()
            hr.close()
            rr = ref.cpu().numpy()
            for a in range(4):
                assert np.array_equal(got[a].numpy()[lo:hi], rr[a, lo:hi])
        h.close()


def test_pipelined_fallback_when_pack_cannot_co_reside(monkeypatch):
    """Without room for a pack block beside a P2P CTA (forced here with
    AFMM_PACK_CORESIDENT=0, read at afmm_p2p_create) the pipelined evaluation
    packs every chunk before the launch: stats.streamed_inputs = 0, same bits."""
    afmm = _afmm()
    bod, T = _setup(n=80000, S=64, seed=9)
    n = bod.shape[1]
    ref, _, _ = _plain(bod, T)
    hb = [bod[a].cpu().pin_memory() for a in range(4)]
    for flag, want in (("0", 0), ("1", 1)):
        monkeypatch.setenv("AFMM_PACK_CORESIDENT", flag)
        h = afmm.P2P(eps2=1e-6)
        h.set_bodies(bod[0], bod[1], bod[2], bod[3])
        h.set_tree(T["leaf_start"], T["leaf_count"], T["u_off"], T["u_idx"])
        got = [torch.full((n,), float("nan")).pin_memory() for _ in range(4)]
        st = h.eval_host_pipelined(*hb, *got, pieces=1)
        assert st["streamed_inputs"] == want
        assert np.array_equal(np.stack([g.numpy() for g in got]), ref)
        h.close()
