"""torch.distributed plumbing for the multi-GPU path.

No arithmetic of the method lives here: these helpers only move the library's
inputs and outputs between ranks (NCCL over NVLink/NVSwitch on B200; gloo on
CPU in the tests).

* packed_bodies(h, device)     -- a4: the library's packed body array as a
                                  tensor: the root packs, one broadcast of it
                                  replicates the bodies (bench.py N > 1).
* replicate(tensors, src)      -- a4: "building the data to send to the GPUs"
                                  (PAPER L16 SIII.C): every rank holds all bodies.
* gather_slices(rows, split)   -- a7: every rank's disjoint output slice to all
                                  ranks (allgatherv as one broadcast per owner);
                                  the paper's blocking copy "into known
                                  locations" (L16 SIII.D).
* open_peer_windows(h, out)    -- a7 fused: every rank's (4, n) output array is
                                  opened in every other rank over CUDA IPC and
                                  registered as a peer window of the library
                                  handle, so the P2P kernel itself stores each
                                  result into all ranks' arrays over NVLink
                                  (no NCCL gather); complete after a barrier.
* allgather_scalar(v, device)  -- a8: per-rank kernel times for the GPU time
                                  (max over GPUs, L20 SVII.A) and the rebalance.
* deliver_chunks(h, stream, src) -- a4 overlapped, caller-driven: after
                                  h.eval_chunked(...) the packed bodies go out
                                  chunk by chunk in the library's delivery order
                                  (afmm_p2p_chunks), each chunk published to the
                                  running kernel (afmm_p2p_publish_chunks) as soon
                                  as it is in place.  (With a library communicator,
                                  P2P(nccl_id=...), eval does this itself over NCCL.)
"""
from __future__ import annotations

import numpy as np
import torch
import torch.distributed as dist


def body_split_from(leaf_split, leaf_start, n):
    """Rank r owns output bodies [body_split[r], body_split[r+1])."""
    ls = np.asarray(leaf_split, np.int64)
    L = len(leaf_start)
    return np.array([n if v >= L else int(leaf_start[v]) for v in ls], np.int64)


class _DeviceArray:
    """A raw device range as a __cuda_array_interface__ object (zero copy)."""

    def __init__(self, ptr, nbytes):
        self.__cuda_array_interface__ = {"shape": (nbytes // 4,), "typestr": "<f4", "data": (int(ptr), False),
                                         "version": 3}


def packed_bodies(h, device):
    """The handle's packed {x, y, z, m} body array (afmm_p2p_bodies_buffer) as a
    float32 CUDA tensor view, for one NCCL broadcast of the packed bodies (a4)."""
    ptr, nbytes = h.bodies_buffer()
    return torch.as_tensor(_DeviceArray(ptr, nbytes), device=device)


def replicate(tensors, src=0):
    for t in tensors:
        dist.broadcast(t, src=src)


def gather_slices(rows, body_split):
    """rows: list of 1-D tensors (length n) owned piecewise by the ranks."""
    world = len(body_split) - 1
    for r in range(world):
        lo, hi = int(body_split[r]), int(body_split[r + 1])
        if hi > lo:
            for row in rows:
                dist.broadcast(row[lo:hi], src=r)


def open_peer_windows(h, out):
    """out: this rank's contiguous (4, n) float32 CUDA tensor (ax, ay, az, phi).
    Exchanges IPC handles (all_gather_object) and registers the peers' rows as
    the handle's peer windows.  Returns a function that unregisters and closes
    them."""
    from . import ipc_close, ipc_export, ipc_import
    if out.dim() != 2 or out.shape[0] != 4 or not out.is_contiguous():
        raise ValueError("out must be a contiguous (4, n) tensor")
    world, rank = dist.get_world_size(), dist.get_rank()
    blobs = [None] * world
    dist.all_gather_object(blobs, ipc_export(out))
    stride = out.shape[1] * out.element_size()
    windows, bases = [], []
    for r in range(world):
        if r == rank:
            continue
        ptr, base = ipc_import(blobs[r])
        bases.append(base)
        windows.append(tuple(ptr + a * stride for a in range(4)))
    h.set_peer_windows(windows)
    dist.barrier()

    def close():
        h.set_peer_windows([])
        for b in bases:
            ipc_close(b)
    return close


def deliver_chunks(h, stream, src=0):
    """Replicate h's packed body array from rank `src` chunk by chunk, after
    h.eval_chunked(...) launched the kernel: the 16-byte trailer first, then the
    chunks in delivery order, each followed by h.publish_chunks(j + 1) on `stream`
    (a torch.cuda.Stream other than the kernel's).  NCCL: device broadcasts on
    `stream`; gloo: staged through host memory (tests on one GPU).
    `stream` must have been ordered after the handle's earlier work (readers of
    the old bodies) BEFORE eval_chunked was called -- ordering it after the
    handle's stream now would wait for the kernel, which waits for the chunks."""
    bounds, order = h.chunks()
    ptr, nbytes = h.bodies_buffer()
    dev = torch.device("cuda", torch.cuda.current_device())
    packed = torch.as_tensor(_DeviceArray(ptr, nbytes), device=dev)    # float32 view, 4 per body + trailer
    n4 = int(bounds[-1]) * 4
    gloo = dist.get_backend() == "gloo"
    rank = dist.get_rank()

    def bcast(view):
        if not gloo:
            dist.broadcast(view, src=src)
            return
        stream.synchronize()
        buf = view.cpu() if rank == src else torch.empty(view.shape, dtype=view.dtype)
        dist.broadcast(buf, src=src)
        if rank != src:
            view.copy_(buf, non_blocking=False)

    with torch.cuda.stream(stream):
        bcast(packed[n4:n4 + 4])
        for j, c in enumerate(order):
            lo, hi = int(bounds[c]) * 4, int(bounds[c + 1]) * 4
            if hi > lo:
                bcast(packed[lo:hi])
            h.publish_chunks(j + 1, stream.cuda_stream)


def allgather_scalar(v: float, device) -> np.ndarray:
    t = torch.tensor([float(v)], dtype=torch.float64, device=device)
    out = [torch.zeros_like(t) for _ in range(dist.get_world_size())]
    dist.all_gather(out, t)
    return np.array([float(o.item()) for o in out])
