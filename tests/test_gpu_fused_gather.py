"""Fused output gather (row a7): the P2P kernel stores every result into every
rank's output arrays (peer windows), so no NCCL gather follows the kernel.

* one process, several handles (ranks) on one GPU, windows = the other
  handles' local arrays: every array ends up holding the whole result,
  bit-identical to a world = 1 evaluation (partition independence, R17);
* two processes on one GPU exchanging CUDA IPC handles through gloo (the
  production path of bench.py at N > 1, dist.open_peer_windows), same check;
* the window API's error statuses."""
import os
import tempfile

import numpy as np
import pytest

import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


def _afmm():
    import paper_conf_ipps_overmanpmm13_b200 as afmm
    return afmm


def _setup(n, S, seed, dist_name="plummer"):
    afmm = _afmm()
    x, y, z, m = synth.make(dist_name, n, seed)
    dev = torch.device("cuda", 0)
    X, Y, Z, M = (torch.from_numpy(v).to(dev) for v in (x, y, z, m))
    t = afmm.GpuTree(0)
    t.build(X, Y, Z, S)
    T = t.copy_out(n)
    b = torch.empty((4, n), device=dev)
    for i, s in enumerate((X, Y, Z, M)):
        t.gather(s, b[i])
    torch.cuda.synchronize()
    t.close()
    return b, T


def _eval(b, T, world, rank, out, eps2=1e-6, windows=None, slice_world=0):
    afmm = _afmm()
    h = afmm.P2P(device=0, rank=rank, world=world, eps2=eps2, slice_world=slice_world)
    h.set_bodies(b[0], b[1], b[2], b[3])
    h.set_tree(T["leaf_start"], T["leaf_count"], T["u_off"], T["u_idx"])
    if windows is not None:
        h.set_peer_windows(windows)
    h.eval(out[0], out[1], out[2], out[3])
    return h


@pytest.mark.parametrize("world", [2, 3, 8])
def test_windows_single_process_bit_identical(world):
    n = 60000
    b, T = _setup(n, 64, 5)
    ref = torch.full((4, n), float("nan"), device="cuda")
    _eval(b, T, 1, 0, ref, slice_world=world).close()        # the same task slicing as the ranks
    outs = [torch.full((4, n), float("nan"), device="cuda") for _ in range(world)]
    hs = []
    for r in range(world):
        peers = [tuple(outs[q][a] for a in range(4)) for q in range(world) if q != r]
        hs.append(_eval(b, T, world, r, outs[r], windows=peers))
    torch.cuda.synchronize()
    R = ref.cpu().numpy()
    assert np.isfinite(R).all()
    for r in range(world):
        np.testing.assert_array_equal(outs[r].cpu().numpy(), R)
    for h in hs:
        h.close()


def test_windows_clear_and_errors():
    afmm = _afmm()
    n = 5000
    b, T = _setup(n, 32, 6)
    own = torch.full((4, n), float("nan"), device="cuda")
    peer = torch.full((4, n), float("nan"), device="cuda")
    h = _eval(b, T, 2, 0, own, windows=[tuple(peer[a] for a in range(4))])
    torch.cuda.synchronize()
    lo, hi = (int(v) for v in (h.stats()["body_lo"], h.stats()["body_hi"]))
    P = peer.cpu().numpy()
    np.testing.assert_array_equal(P[:, lo:hi], own.cpu().numpy()[:, lo:hi])
    assert np.isnan(P[:, hi:]).all() and np.isnan(P[:, :lo]).all()     # only this rank's slice
    # cleared windows: the peer is no longer written
    peer.fill_(float("nan"))
    h.set_peer_windows([])
    h.eval(own[0], own[1], own[2], own[3])
    torch.cuda.synchronize()
    assert np.isnan(peer.cpu().numpy()).all()
    with pytest.raises(afmm.AfmmError):
        h.set_peer_windows([tuple(peer[a] for a in range(4))] * 8)      # > 7 peers
    with pytest.raises(afmm.AfmmError):
        h.set_peer_windows([(peer[0], peer[1], peer[2], 0)])           # null pointer
    h.close()


def _ipc_worker(rank, world, port, path, n, S, seed):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    from paper_conf_ipps_overmanpmm13_b200 import dist as pdist
    b, T = _setup(n, S, seed)
    out = torch.full((4, n), float("nan"), device="cuda")
    afmm = _afmm()
    h = afmm.P2P(device=0, rank=rank, world=world, eps2=1e-6)
    h.set_bodies(b[0], b[1], b[2], b[3])
    h.set_tree(T["leaf_start"], T["leaf_count"], T["u_off"], T["u_idx"])
    close = pdist.open_peer_windows(h, out)
    h.eval(out[0], out[1], out[2], out[3])
    torch.cuda.synchronize()
    dist.barrier()                    # every rank's kernel (and its peer stores) has completed
    np.save(os.path.join(path, f"out{rank}.npy"), out.cpu().numpy())
    dist.barrier()
    close()
    h.close()
    dist.destroy_process_group()


def test_ipc_two_processes_same_gpu():
    import socket
    import torch.multiprocessing as mp
    n, S, seed, world = 80000, 96, 7, 2
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    with tempfile.TemporaryDirectory() as d:
        mp.spawn(_ipc_worker, args=(world, port, d, n, S, seed), nprocs=world, join=True)
        outs = [np.load(os.path.join(d, f"out{r}.npy")) for r in range(world)]
    b, T = _setup(n, S, seed)
    ref = torch.full((4, n), float("nan"), device="cuda")
    _eval(b, T, 1, 0, ref, slice_world=world).close()
    R = ref.cpu().numpy()
    assert np.isfinite(R).all()
    for r in range(world):
        np.testing.assert_array_equal(outs[r], R)
