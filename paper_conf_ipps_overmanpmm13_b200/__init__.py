"""Thin ctypes binding of libafmm_p2p.so (include/afmm_p2p.h, include/afmm_tree.h).

Argument marshalling only: every step of the near-field path (packing, tree
construction, U-lists, the P2P kernel) runs in the CUDA library.  There is no
CPU fallback: importing this package raises if the shared library is missing,
and every call raises ``AfmmError`` on a non-zero status.

Names follow the C ABI: ``create``, ``set_bodies``, ``set_tree``, ``eval`` ...
of AFMM P2P (Overman et al., IPDPSW 2013, PAPER.md L12 SI.C / L16 SIII.C).
Tensors are ``torch`` CUDA tensors (device pointers) or numpy arrays (host
pointers) -- torch is only the device-memory / stream provider.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("AFMM_LIB_OVERRIDE") or os.path.join(_HERE, "libafmm_p2p.so")  # override: tools/tune only

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} not built: run `make` (or __graft_entry__.build()) first; "
                      "there is no CPU fallback for the AFMM P2P path")
_lib = C.CDLL(LIB_PATH)

MAX_LEAF = 1 << 30     # AFMM_MAX_LEAF of include/afmm_p2p.h
AFMM_OK, AFMM_EINVAL, AFMM_ESTATE, AFMM_ENOMEM, AFMM_ECUDA, AFMM_ENCCL, AFMM_ENOTSUP = 0, -1, -2, -3, -4, -5, -6
_STATUS = {0: "AFMM_OK", -1: "AFMM_EINVAL", -2: "AFMM_ESTATE", -3: "AFMM_ENOMEM", -4: "AFMM_ECUDA",
           -5: "AFMM_ENCCL", -6: "AFMM_ENOTSUP"}
N_BUCKETS = 8


class AfmmError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{_STATUS.get(status, status)}: {msg}")
        self.status = status


class Config(C.Structure):
    _fields_ = [("device", C.c_int), ("rank", C.c_int), ("world", C.c_int), ("G", C.c_float),
                ("eps2", C.c_float), ("max_leaf", C.c_int), ("stream", C.c_void_p), ("law", C.c_int),
                ("mu", C.c_float), ("slice_world", C.c_int), ("nccl_id", C.c_void_p), ("comm_sms", C.c_int)]


LAW_GRAVITY, LAW_STOKESLET = 0, 1


class Stats(C.Structure):
    _fields_ = [("kernel_ms", C.c_double), ("interactions_total", C.c_longlong),
                ("interactions_rank", C.c_longlong), ("leaf_lo", C.c_longlong),
                ("leaf_hi", C.c_longlong), ("body_lo", C.c_longlong), ("body_hi", C.c_longlong),
                ("n_work_items", C.c_int), ("n_launches", C.c_int),
                ("bucket_interactions", C.c_longlong * N_BUCKETS), ("zero_copy", C.c_int),
                ("input_graph", C.c_int), ("streamed_inputs", C.c_int), ("chunked_bodies", C.c_int),
                ("kernel_ms_max", C.c_double)]

    def as_dict(self):
        d = {f: getattr(self, f) for f, _ in self._fields_ if f != "bucket_interactions"}
        d["bucket_interactions"] = list(self.bucket_interactions)
        return d


_p, _i, _ll, _d = C.c_void_p, C.c_int, C.c_longlong, C.c_double


def _sig(name, res, *args):
    if os.environ.get("AFMM_LIB_OVERRIDE") and not hasattr(_lib, name):
        return None                       # tools/tune: an older build without this entry point
    f = getattr(_lib, name)
    f.restype = res
    f.argtypes = list(args)
    return f


_sig("afmm_p2p_config_init", _i, C.POINTER(Config))
_sig("afmm_p2p_create", _i, C.POINTER(Config), C.POINTER(_p))
_sig("afmm_p2p_set_bodies", _i, _p, _ll, _p, _p, _p, _p)
_sig("afmm_p2p_interactions", _i, _p, C.POINTER(_ll), C.POINTER(_ll))
_sig("afmm_p2p_set_bodies_deferred", _i, _p, _ll, _p, _p, _p, _p)
_sig("afmm_p2p_set_bodies_host", _i, _p, _ll, _p, _p, _p, _p)
_sig("afmm_p2p_bodies_buffer", _i, _p, C.POINTER(_p), C.POINTER(_ll))
_sig("afmm_p2p_set_bodies_stokeslet", _i, _p, _ll, _p, _p, _p, _p, _p, _p)
_sig("afmm_p2p_set_tree", _i, _p, _i, _p, _p, _p, _p)
_sig("afmm_p2p_set_partition", _i, _p, _p)
_sig("afmm_p2p_set_tree_device", _i, _p, _i, _p, _p, _p, _p)
_sig("afmm_tree_device_arrays", _i, _p, C.POINTER(_p), C.POINTER(_p), C.POINTER(_p), C.POINTER(_p), C.POINTER(_p))
_sig("afmm_p2p_get_partition", _i, _p, _p, _p)
_sig("afmm_p2p_rebalance", _i, _p, _p, _d, C.POINTER(_i))
_sig("afmm_p2p_eval", _i, _p, _p, _p, _p, _p, C.POINTER(Stats))
_sig("afmm_p2p_eval_host", _i, _p, _p, _p, _p, _p, C.POINTER(Stats))
_sig("afmm_p2p_eval_host_pipelined", _i, _p, _ll, _p, _p, _p, _p, _p, _p, _p, _p, _i, C.POINTER(Stats))
_sig("afmm_p2p_stats_get", _i, _p, C.POINTER(Stats))
_sig("afmm_p2p_set_peer_windows", _i, _p, _i, _p)
_sig("afmm_p2p_nccl_id", _i, _p)
_sig("afmm_p2p_chunks", _i, _p, C.POINTER(_i), _p, _p)
_sig("afmm_p2p_worklist", _i, _p, _p, _ll, C.POINTER(_ll), _p, _ll, C.POINTER(_ll))
_sig("afmm_p2p_eval_chunked", _i, _p, _p, _p, _p, _p)
_sig("afmm_p2p_publish_chunks", _i, _p, _i, _p)


class IpcHandle(C.Structure):
    _fields_ = [("handle", C.c_ubyte * 64), ("offset", C.c_longlong)]


_sig("afmm_ipc_export", _i, _p, C.POINTER(IpcHandle))
_sig("afmm_ipc_import", _i, C.POINTER(IpcHandle), C.POINTER(_p), C.POINTER(_p))
_sig("afmm_ipc_close", _i, _p)
_sig("afmm_p2p_stream", _p, _p)
_sig("afmm_p2p_kernel_times", _i, _p, _i, _p)
_sig("afmm_p2p_destroy", None, _p)
_sig("afmm_p2p_last_error", C.c_char_p, _p)
_sig("afmm_interactions", _i, _i, _p, _p, _p, _p)
_sig("afmm_partition_literal", _i, _i, _p, _i, _p)
_sig("afmm_partition_weighted", _i, _i, _p, _i, _p)
_sig("afmm_partition_rebalance", _i, _i, _p, _p, _i, _p, _p, _d, _p, C.POINTER(_i))
_sig("afmm_cost_fit", _i, _i, _p, _p, _p)
_sig("afmm_p2p_set_cost_coef", _i, _p, _p)
_sig("afmm_kick", _i, _ll, _p, _p, _p, _p, _p, _p, C.c_float, _p)
_sig("afmm_drift", _i, _ll, _p, _p, _p, _p, _p, _p, C.c_float, _p)
_sig("afmm_kick_drift", _i, _ll, _p, _p, _p, _p, _p, _p, _p, _p, _p, C.c_float, C.c_float, _p)
_sig("afmm_fp32_peak", _i, _i, C.POINTER(_d), C.POINTER(_d), C.POINTER(_d))
_sig("afmm_version", C.c_char_p)
_sig("afmm_launch_count", C.c_longlong)
_sig("afmm_tree_create", _i, _i, _p, C.POINTER(_p))
_sig("afmm_tree_build", _i, _p, _ll, _p, _p, _p, _i, _i, _p, _i)
_sig("afmm_tree_enforce", _i, _p, _ll, _p, _p, _p, _i)
_sig("afmm_tree_farfield_counts", _i, _p, _p)
_sig("afmm_tree_info", _i, _p, C.POINTER(_i), C.POINTER(_ll), _p, C.POINTER(_i), C.POINTER(_i),
     C.POINTER(_ll))
_sig("afmm_tree_counters", _i, _p, C.POINTER(_ll), C.POINTER(_ll))
_sig("afmm_tree_copy_out", _i, _p, _p, _p, _p, _p, _p, _p, _p)
_sig("afmm_tree_gather", _i, _p, _p, _p)
_sig("afmm_tree_gather_rows", _i, _p, _i, _p, _p)
_sig("afmm_tree_scatter", _i, _p, _p, _p)
_sig("afmm_tree_destroy", None, _p)
_sig("afmm_tree_last_error", C.c_char_p, _p)

class LbConfig(C.Structure):
    _fields_ = [("S_init", C.c_int), ("S_min", C.c_int), ("S_max", C.c_int), ("dS", C.c_int),
                ("balance_rel", C.c_double), ("observe_rel", C.c_double)]


LB_SEARCH, LB_INCREMENTAL, LB_OBSERVATION = 0, 1, 2
LB_KEEP, LB_REBUILD, LB_ENFORCE, LB_FINE = 0, 1, 2, 3
_sig("afmm_lb_config_init", _i, C.POINTER(LbConfig))
_sig("afmm_lb_create", _i, C.POINTER(LbConfig), C.POINTER(_p))
_sig("afmm_lb_step", _i, _p, _d, _d, C.POINTER(_i), C.POINTER(_i))
_sig("afmm_lb_predicted", _i, _p, _d, C.POINTER(_i))
_sig("afmm_lb_state", _i, _p, C.POINTER(_i), C.POINTER(_i), C.POINTER(_d))
_sig("afmm_lb_predict", _i, _p, _p, C.POINTER(_d), C.POINTER(_d), C.POINTER(_d))
_sig("afmm_lb_destroy", None, _p)


class FgResult(C.Structure):
    _fields_ = [("direction", C.c_int), ("groups_tried", C.c_int), ("groups_applied", C.c_int),
                ("nodes_changed", C.c_longlong), ("t_before", C.c_double), ("t_after", C.c_double),
                ("t_cpu_after", C.c_double), ("t_gpu_after", C.c_double)]


TREE_ENFORCE, TREE_KEEP = 1, 2
COLLAPSE, PUSHDOWN = 1, 2
_sig("afmm_tree_rebuild", _i, _p, _ll, _p, _p, _p, _i, _i, _i, _p, _p, _p)
_sig("afmm_tree_nodes", _i, _p, _p, _p, _p)
_sig("afmm_fine_grained", _i, _p, _ll, _p, _p, _p, _i, _p, _i, _d, _i, C.POINTER(FgResult))

# every symbol include/*.h declares (checked by tests/test_abi.py)
EXPORTED = ["afmm_p2p_config_init", "afmm_p2p_create", "afmm_p2p_set_bodies",
            "afmm_p2p_set_bodies_host", "afmm_p2p_bodies_buffer", "afmm_p2p_set_tree",
            "afmm_p2p_set_bodies_stokeslet",
            "afmm_p2p_set_partition", "afmm_p2p_get_partition", "afmm_p2p_rebalance",
            "afmm_p2p_set_tree_device", "afmm_tree_device_arrays",
            "afmm_p2p_eval", "afmm_p2p_eval_host", "afmm_p2p_stats_get", "afmm_p2p_stream", "afmm_p2p_set_bodies_deferred", "afmm_p2p_interactions",
            "afmm_p2p_kernel_times",
            "afmm_p2p_destroy", "afmm_p2p_last_error", "afmm_interactions",
            "afmm_partition_literal", "afmm_partition_weighted", "afmm_partition_rebalance",
            "afmm_cost_fit", "afmm_p2p_set_cost_coef", "afmm_kick", "afmm_drift", "afmm_kick_drift",
            "afmm_fp32_peak", "afmm_version",
            "afmm_tree_create", "afmm_tree_build", "afmm_tree_enforce", "afmm_tree_info", "afmm_tree_counters",
            "afmm_tree_farfield_counts", "afmm_lb_config_init", "afmm_lb_create", "afmm_lb_step",
            "afmm_lb_predicted", "afmm_lb_state", "afmm_lb_destroy", "afmm_tree_copy_out",
            "afmm_tree_gather", "afmm_tree_scatter", "afmm_tree_destroy", "afmm_tree_last_error",
            "afmm_tree_rebuild", "afmm_tree_nodes", "afmm_fine_grained", "afmm_p2p_eval_host_pipelined",
            "afmm_p2p_set_peer_windows", "afmm_ipc_export", "afmm_ipc_import", "afmm_ipc_close",
            "afmm_tree_gather_rows", "afmm_p2p_nccl_id", "afmm_p2p_chunks", "afmm_p2p_eval_chunked",
            "afmm_p2p_publish_chunks", "afmm_launch_count", "afmm_lb_predict", "afmm_p2p_worklist"]


def ipc_export(dev_ptr):
    """afmm_ipc_export: bytes (64-B cudaIpcMemHandle of the base allocation +
    8-B offset) describing a device pointer (int) or CUDA tensor."""
    h = IpcHandle()
    ptr = dev_ptr.data_ptr() if hasattr(dev_ptr, "data_ptr") else int(dev_ptr)
    st = _lib.afmm_ipc_export(C.c_void_p(ptr), C.byref(h))
    if st:
        raise AfmmError(st, "afmm_ipc_export")
    return bytes(C.string_at(C.addressof(h), C.sizeof(h)))


def ipc_import(blob):
    """afmm_ipc_import: (device pointer, base) in this process; close with ipc_close(base)."""
    h = IpcHandle.from_buffer_copy(blob)
    p, b = _p(), _p()
    st = _lib.afmm_ipc_import(C.byref(h), C.byref(p), C.byref(b))
    if st:
        raise AfmmError(st, "afmm_ipc_import")
    return p.value, b.value


def ipc_close(base):
    st = _lib.afmm_ipc_close(C.c_void_p(base))
    if st:
        raise AfmmError(st, "afmm_ipc_close")


def version() -> str:
    return _lib.afmm_version().decode()


def launch_count() -> int:
    """afmm_launch_count: this library's kernels launched so far in this process."""
    return int(_lib.afmm_launch_count())


def nccl_id() -> bytes:
    """afmm_p2p_nccl_id: a new 128-byte ncclUniqueId (rank 0) for P2P(nccl_id=...)."""
    buf = C.create_string_buffer(128)
    st = _lib.afmm_p2p_nccl_id(buf)
    if st:
        raise AfmmError(st, "afmm_p2p_nccl_id")
    return buf.raw


def _np(a, dt):
    return np.ascontiguousarray(a, dtype=dt)


def _ptr(a):
    """Raw pointer of a numpy array or a torch tensor (host or device)."""
    if a is None:
        return None
    if isinstance(a, np.ndarray):
        return a.ctypes.data
    return a.data_ptr()


def _check_host_tensor(t, n):
    import torch
    if t.is_cuda or t.dtype != torch.float32 or not t.is_contiguous() or t.shape[0] != n:
        raise TypeError("host tensors must be contiguous float32 CPU tensors of length n")


def _is_device(a) -> bool:
    return not isinstance(a, np.ndarray) and getattr(a, "is_cuda", False)


# ------------------------------------------------------------------ host-only helpers

def interactions(leaf_count, u_off, u_idx) -> np.ndarray:
    """Interactions(t) = n_t * sum_{s in U(t)} n_s (PAPER L16 SIII.C)."""
    lc, uo, ui = _np(leaf_count, np.int32), _np(u_off, np.int64), _np(u_idx, np.int32)
    out = np.empty(lc.shape[0], np.int64)
    st = _lib.afmm_interactions(lc.shape[0], _ptr(lc), _ptr(uo), _ptr(ui), _ptr(out))
    if st:
        raise AfmmError(st, "afmm_interactions")
    return out


def partition_literal(I, G: int) -> np.ndarray:
    """Literal greedy split of PAPER L16 SIII.C -> leaf_split[G+1]."""
    I = _np(I, np.int64)
    out = np.empty(G + 1, np.int64)
    st = _lib.afmm_partition_literal(I.shape[0], _ptr(I), int(G), _ptr(out))
    if st:
        raise AfmmError(st, "afmm_partition_literal")
    return out


def partition_weighted(w, G: int) -> np.ndarray:
    w = _np(w, np.float64)
    out = np.empty(G + 1, np.int64)
    st = _lib.afmm_partition_weighted(w.shape[0], _ptr(w), int(G), _ptr(out))
    if st:
        raise AfmmError(st, "afmm_partition_weighted")
    return out


def partition_rebalance(leaf_count, I, cur_split, rank_ms, threshold=0.02):
    """Host-only rebalance rule (see afmm_partition_rebalance) -> (new_split, changed)."""
    lc, I = _np(leaf_count, np.int32), _np(I, np.int64)
    cs, rm = _np(cur_split, np.int64), _np(rank_ms, np.float64)
    G = cs.shape[0] - 1
    out = np.empty(G + 1, np.int64)
    ch = _i()
    st = _lib.afmm_partition_rebalance(lc.shape[0], _ptr(lc), _ptr(I), G, _ptr(cs), _ptr(rm),
                                       float(threshold), _ptr(out), C.byref(ch))
    if st:
        raise AfmmError(st, "afmm_partition_rebalance")
    return out, bool(ch.value)


def cost_fit(bucket_inter, rank_ms):
    """Per-bucket cost coefficients (afmm_cost_fit); bucket_inter: [G, 8]."""
    B = _np(bucket_inter, np.float64).reshape(-1, N_BUCKETS)
    r = _np(rank_ms, np.float64)
    out = np.empty(N_BUCKETS, np.float64)
    st = _lib.afmm_cost_fit(B.shape[0], _ptr(B), _ptr(r), _ptr(out))
    if st:
        raise AfmmError(st, "afmm_cost_fit")
    return out


def kick(vx, vy, vz, ax, ay, az, h, stream=None):
    """Leapfrog kick v <- v + h a on device tensors (afmm_kick)."""
    st = _lib.afmm_kick(int(vx.shape[0]), _ptr(vx), _ptr(vy), _ptr(vz), _ptr(ax), _ptr(ay), _ptr(az),
                        float(h), stream)
    if st:
        raise AfmmError(st, "afmm_kick")


def drift(x, y, z, vx, vy, vz, dt, stream=None):
    """Leapfrog drift x <- x + dt v on device tensors (afmm_drift)."""
    st = _lib.afmm_drift(int(x.shape[0]), _ptr(x), _ptr(y), _ptr(z), _ptr(vx), _ptr(vy), _ptr(vz),
                         float(dt), stream)
    if st:
        raise AfmmError(st, "afmm_drift")


def kick_drift(x, y, z, vx, vy, vz, ax, ay, az, h, dt, stream=None):
    """Kick then drift in one kernel (afmm_kick_drift; bit-identical to kick + drift)."""
    st = _lib.afmm_kick_drift(int(x.shape[0]), _ptr(x), _ptr(y), _ptr(z), _ptr(vx), _ptr(vy), _ptr(vz), _ptr(ax),
                              _ptr(ay), _ptr(az), float(h), float(dt), stream)
    if st:
        raise AfmmError(st, "afmm_kick_drift")


def fp32_peak(device: int = 0):
    """Measured FP32 FFMA / FFMA2 TFLOP/s and the SM clock (MHz) on `device`."""
    a, b, c = _d(), _d(), _d()
    st = _lib.afmm_fp32_peak(int(device), C.byref(a), C.byref(b), C.byref(c))
    if st:
        raise AfmmError(st, "afmm_fp32_peak")
    return {"ffma_tflops": a.value, "ffma2_tflops": b.value, "sm_mhz": c.value}


# ------------------------------------------------------------------ P2P handle

class P2P:
    """One afmm_p2p handle (one per rank / GPU)."""

    def __init__(self, device=0, rank=0, world=1, G=1.0, eps2=0.0, max_leaf=None, stream=None,
                 law=LAW_GRAVITY, mu=1.0, slice_world=0, nccl_id=None, comm_sms=0):
        cfg = Config()
        _lib.afmm_p2p_config_init(C.byref(cfg))
        cfg.device, cfg.rank, cfg.world = int(device), int(rank), int(world)
        cfg.G, cfg.eps2 = float(G), float(eps2)
        if max_leaf is not None:
            cfg.max_leaf = int(max_leaf)
        cfg.stream = stream
        cfg.law, cfg.mu = int(law), float(mu)
        cfg.slice_world = int(slice_world)
        idbuf = None
        if nccl_id is not None:
            if len(nccl_id) != 128:
                raise ValueError("nccl_id must be the 128-byte id of afmm_p2p_nccl_id")
            idbuf = C.create_string_buffer(bytes(nccl_id), 128)
            cfg.nccl_id = C.cast(idbuf, C.c_void_p)
        cfg.comm_sms = int(comm_sms)
        h = _p()
        st = _lib.afmm_p2p_create(C.byref(cfg), C.byref(h))
        if st:
            raise AfmmError(st, "afmm_p2p_create")
        self._h = h
        self.world, self.rank, self.device = world, rank, device

    def _check(self, st, what):
        if st:
            raise AfmmError(st, f"{what}: {_lib.afmm_p2p_last_error(self._h).decode()}")

    def close(self):
        if getattr(self, "_h", None) and _lib is not None:   # _lib is None at interpreter exit
            _lib.afmm_p2p_destroy(self._h)
        self._h = None

    __del__ = close

    @property
    def stream(self):
        return _lib.afmm_p2p_stream(self._h)

    def set_bodies(self, x, y, z, m, n=None):
        """Bodies in tree order.  torch CUDA tensors -> afmm_p2p_set_bodies;
        numpy arrays -> afmm_p2p_set_bodies_host; all None with n -> allocate only."""
        if x is None:
            self._check(_lib.afmm_p2p_set_bodies(self._h, int(n), None, None, None, None),
                        "afmm_p2p_set_bodies")
            return
        n = int(x.shape[0])
        if _is_device(x):
            self._check(_lib.afmm_p2p_set_bodies(self._h, n, _ptr(x), _ptr(y), _ptr(z), _ptr(m)),
                        "afmm_p2p_set_bodies")
        elif not isinstance(x, np.ndarray):          # torch CPU (e.g. pinned) tensors
            for v in (x, y, z, m):
                _check_host_tensor(v, n)
            self._check(_lib.afmm_p2p_set_bodies_host(self._h, n, _ptr(x), _ptr(y), _ptr(z), _ptr(m)),
                        "afmm_p2p_set_bodies_host")
        else:
            x, y, z, m = (_np(v, np.float32) for v in (x, y, z, m))
            self._check(_lib.afmm_p2p_set_bodies_host(self._h, n, _ptr(x), _ptr(y), _ptr(z), _ptr(m)),
                        "afmm_p2p_set_bodies_host")

    def set_bodies_deferred(self, x, y, z, m):
        """afmm_p2p_set_bodies_deferred (torch CUDA tensors, root of a library
        communicator): packed chunk by chunk inside the next eval; the tensors must
        stay alive and unchanged until that eval's stream work completes."""
        if not _is_device(x):
            raise ValueError("set_bodies_deferred takes CUDA tensors")
        self._check(_lib.afmm_p2p_set_bodies_deferred(self._h, int(x.shape[0]), _ptr(x), _ptr(y), _ptr(z), _ptr(m)),
                    "afmm_p2p_set_bodies_deferred")

    def set_bodies_stokeslet(self, x, y, z, fx, fy, fz):
        """Stokeslet bodies: torch CUDA tensors (device pointers), tree order."""
        self._check(_lib.afmm_p2p_set_bodies_stokeslet(self._h, int(x.shape[0]), *[_ptr(a) for a in
                                                                                  (x, y, z, fx, fy, fz)]),
                    "afmm_p2p_set_bodies_stokeslet")

    def bodies_buffer(self):
        p, b = _p(), _ll()
        self._check(_lib.afmm_p2p_bodies_buffer(self._h, C.byref(p), C.byref(b)), "afmm_p2p_bodies_buffer")
        return p.value, b.value

    def set_tree(self, leaf_start, leaf_count, u_off, u_idx):
        ls, lc = _np(leaf_start, np.int32), _np(leaf_count, np.int32)
        uo, ui = _np(u_off, np.int64), _np(u_idx, np.int32)
        self._check(_lib.afmm_p2p_set_tree(self._h, ls.shape[0], _ptr(ls), _ptr(lc), _ptr(uo), _ptr(ui)),
                    "afmm_p2p_set_tree")

    def set_tree_device(self, n_leaves, leaf_start, leaf_count, u_off, u_idx):
        """Tree ingest from device pointers (ints) or torch CUDA tensors."""
        ptr = lambda a: a if isinstance(a, int) else _ptr(a)  # noqa: E731
        self._check(_lib.afmm_p2p_set_tree_device(self._h, int(n_leaves), ptr(leaf_start), ptr(leaf_count),
                                                  ptr(u_off), ptr(u_idx)), "afmm_p2p_set_tree_device")

    def set_partition(self, leaf_split=None):
        ls = None if leaf_split is None else _np(leaf_split, np.int64)
        self._check(_lib.afmm_p2p_set_partition(self._h, _ptr(ls)), "afmm_p2p_set_partition")

    def set_cost_coef(self, coef=None):
        c = None if coef is None else _np(coef, np.float64)
        self._check(_lib.afmm_p2p_set_cost_coef(self._h, _ptr(c)), "afmm_p2p_set_cost_coef")

    def get_partition(self):
        ls = np.empty(self.world + 1, np.int64)
        bs = np.empty(self.world + 1, np.int64)
        self._check(_lib.afmm_p2p_get_partition(self._h, _ptr(ls), _ptr(bs)), "afmm_p2p_get_partition")
        return ls, bs

    def rebalance(self, rank_ms, threshold=0.02) -> bool:
        r = _np(rank_ms, np.float64)
        ch = _i()
        self._check(_lib.afmm_p2p_rebalance(self._h, _ptr(r), float(threshold), C.byref(ch)),
                    "afmm_p2p_rebalance")
        return bool(ch.value)

    def eval(self, ax, ay, az, phi, stats=False):
        """Outputs: torch CUDA tensors (async; stats forces a sync) or numpy
        arrays (blocking, afmm_p2p_eval_host)."""
        s = Stats()
        sp = C.byref(s) if stats else None
        if _is_device(ax):
            self._check(_lib.afmm_p2p_eval(self._h, _ptr(ax), _ptr(ay), _ptr(az), _ptr(phi), sp),
                        "afmm_p2p_eval")
        else:
            for a in (ax, ay, az, phi):
                if isinstance(a, np.ndarray):
                    if not (a.dtype == np.float32 and a.flags.c_contiguous):
                        raise TypeError("host outputs must be contiguous float32 arrays")
                else:
                    _check_host_tensor(a, int(a.shape[0]))
            sp = C.byref(s)
            self._check(_lib.afmm_p2p_eval_host(self._h, _ptr(ax), _ptr(ay), _ptr(az), _ptr(phi), sp),
                        "afmm_p2p_eval_host")
        return s.as_dict() if (stats or not _is_device(ax)) else None

    def set_peer_windows(self, windows):
        """afmm_p2p_set_peer_windows: windows = list of (ax, ay, az, phi) device
        pointers (ints) or CUDA tensors of n fp32 each; [] clears."""
        flat = []
        for w in windows:
            if len(w) != 4:
                raise ValueError("a window is (ax, ay, az, phi)")
            flat += [a.data_ptr() if hasattr(a, "data_ptr") else int(a) for a in w]
        arr = (C.c_void_p * max(1, len(flat)))(*flat)
        self._check(_lib.afmm_p2p_set_peer_windows(self._h, len(windows), arr if flat else None),
                    "afmm_p2p_set_peer_windows")

    def eval_host_pipelined(self, x, y, z, m, ax, ay, az, phi, pieces=8):
        """afmm_p2p_eval_host_pipelined: host inputs (tree order) -> host outputs,
        transfers overlapped with the kernel pieces.  Host tensors or numpy
        float32 arrays (pinned torch tensors for the overlap)."""
        arrs = (x, y, z, m, ax, ay, az, phi)
        n = int(x.shape[0])
        for a in arrs:
            if _is_device(a):
                raise TypeError("eval_host_pipelined takes host arrays")
            if isinstance(a, np.ndarray):
                if not (a.dtype == np.float32 and a.flags.c_contiguous and a.shape[0] == n):
                    raise TypeError("host arrays must be contiguous float32 of length n")
            else:
                _check_host_tensor(a, n)
        s = Stats()
        self._check(_lib.afmm_p2p_eval_host_pipelined(self._h, n, *[_ptr(a) for a in arrs], int(pieces), C.byref(s)),
                    "afmm_p2p_eval_host_pipelined")
        return s.as_dict()

    def chunks(self):
        """afmm_p2p_chunks: (bounds[K+1], order[K]) of the chunked body delivery."""
        K = _i()
        self._check(_lib.afmm_p2p_chunks(self._h, C.byref(K), None, None), "afmm_p2p_chunks")
        b = np.empty(K.value + 1, np.int64)
        o = np.empty(K.value, np.int32)
        self._check(_lib.afmm_p2p_chunks(self._h, C.byref(K), _ptr(b), _ptr(o)), "afmm_p2p_chunks")
        return b, o

    def worklist(self):
        """afmm_p2p_worklist: (tasks[nt, 8], segs[ns, 2]) int32, in dispatch order."""
        nt, ns = _ll(), _ll()
        self._check(_lib.afmm_p2p_worklist(self._h, None, 0, C.byref(nt), None, 0, C.byref(ns)), "afmm_p2p_worklist")
        t = np.empty((nt.value, 8), np.int32)
        s = np.empty((ns.value, 2), np.int32)
        self._check(_lib.afmm_p2p_worklist(self._h, _ptr(t), nt.value, C.byref(nt), _ptr(s), ns.value, C.byref(ns)),
                    "afmm_p2p_worklist")
        return t, s

    def eval_chunked(self, ax, ay, az, phi):
        """afmm_p2p_eval_chunked: launch before the bodies arrive (device outputs, async)."""
        self._check(_lib.afmm_p2p_eval_chunked(self._h, _ptr(ax), _ptr(ay), _ptr(az), _ptr(phi)),
                    "afmm_p2p_eval_chunked")

    def publish_chunks(self, count, stream=None):
        """afmm_p2p_publish_chunks: the first `count` chunks of the delivery order are in
        place once `stream` (cudaStream_t int, None = the handle's stream) reaches this."""
        self._check(_lib.afmm_p2p_publish_chunks(self._h, int(count), stream), "afmm_p2p_publish_chunks")

    def kernel_times(self, max_count=64):
        """Kernel ms of the last <= 64 evals (oldest first); synchronises."""
        buf = np.empty(max(1, max_count), np.float64)
        cnt = _lib.afmm_p2p_kernel_times(self._h, int(max_count), _ptr(buf))
        if cnt < 0:
            self._check(cnt, "afmm_p2p_kernel_times")
        return buf[:cnt].copy()

    def interactions(self):
        """(total, this rank's) interactions of the current tree (afmm_p2p_interactions; no sync)."""
        t, r = _ll(), _ll()
        self._check(_lib.afmm_p2p_interactions(self._h, C.byref(t), C.byref(r)), "afmm_p2p_interactions")
        return t.value, r.value

    def stats(self):
        s = Stats()
        self._check(_lib.afmm_p2p_stats_get(self._h, C.byref(s)), "afmm_p2p_stats_get")
        return s.as_dict()


# ------------------------------------------------------------------ GPU tree builder

class GpuTree:
    """afmm_tree handle: adaptive octree + U-list built on the GPU."""

    def __init__(self, device=0, stream=None):
        h = _p()
        st = _lib.afmm_tree_create(int(device), stream, C.byref(h))
        if st:
            raise AfmmError(st, "afmm_tree_create")
        self._h = h

    def _check(self, st, what):
        if st:
            raise AfmmError(st, f"{what}: {_lib.afmm_tree_last_error(self._h).decode()}")

    def close(self):
        if getattr(self, "_h", None) and _lib is not None:
            _lib.afmm_tree_destroy(self._h)
        self._h = None

    __del__ = close

    def build(self, x, y, z, S, domain=None):
        """x, y, z: torch CUDA float32 tensors (input order).  domain=(lo[3], k) fixes it."""
        lo = None
        k = 0
        fixed = 0
        if domain is not None:
            lo = _np(domain[0], np.float64)
            k = int(domain[1])
            fixed = 1
        self._check(_lib.afmm_tree_build(self._h, int(x.shape[0]), _ptr(x), _ptr(y), _ptr(z), int(S),
                                         fixed, _ptr(lo), k), "afmm_tree_build")
        return self.info()

    def enforce(self, x, y, z, S):
        """Enforce_S on the last build for moved bodies (afmm_tree_enforce)."""
        self._check(_lib.afmm_tree_enforce(self._h, int(x.shape[0]), _ptr(x), _ptr(y), _ptr(z), int(S)),
                    "afmm_tree_enforce")
        return self.info()

    def rebuild(self, x, y, z, S, mode=TREE_KEEP, edits=()):
        """afmm_tree_rebuild: previous structure (TREE_KEEP) or Enforce_S rule
        (TREE_ENFORCE), then (level, prefix, COLLAPSE|PUSHDOWN) edits."""
        lev = _np([e[0] for e in edits] or [0], np.int32)
        pre = _np([e[1] for e in edits] or [0], np.uint64)
        act = _np([e[2] for e in edits] or [0], np.int32)
        self._check(_lib.afmm_tree_rebuild(self._h, int(x.shape[0]), _ptr(x), _ptr(y), _ptr(z), int(S), int(mode),
                                           len(edits), _ptr(lev), _ptr(pre), _ptr(act)), "afmm_tree_rebuild")
        return self.info()

    def nodes(self):
        """All nodes of the last build: level, prefix, nchild (numpy)."""
        nn = self.info()["n_nodes"]
        out = {"level": np.empty(nn, np.int32), "prefix": np.empty(nn, np.uint64), "nchild": np.empty(nn, np.int32)}
        self._check(_lib.afmm_tree_nodes(self._h, _ptr(out["level"]), _ptr(out["prefix"]), _ptr(out["nchild"])),
                    "afmm_tree_nodes")
        return out

    def fine_grained(self, x, y, z, S, coef, direction=0, group_frac=0.05, max_groups=16):
        """FineGrainedOptimize (afmm_fine_grained, L20 SVI.B) -> result dict."""
        c = _np(coef, np.float64)
        if c.shape != (6,):
            raise ValueError("coef must hold 6 values (P2M, M2M, M2L, L2L, L2P, P2P)")
        r = FgResult()
        self._check(_lib.afmm_fine_grained(self._h, int(x.shape[0]), _ptr(x), _ptr(y), _ptr(z), int(S), _ptr(c),
                                           int(direction), float(group_frac), int(max_groups), C.byref(r)),
                    "afmm_fine_grained")
        return {k: getattr(r, k) for k, _ in FgResult._fields_}

    def info(self):
        L, nnz, k, ml, nn = _i(), _ll(), _i(), _i(), _ll()
        lo = np.empty(3)
        self._check(_lib.afmm_tree_info(self._h, C.byref(L), C.byref(nnz), _ptr(lo), C.byref(k),
                                        C.byref(ml), C.byref(nn)), "afmm_tree_info")
        return {"n_leaves": L.value, "nnz": nnz.value, "lo": lo, "k": k.value,
                "max_level": ml.value, "n_nodes": nn.value}

    def counters(self):
        """{'graph_launches', 'sort_fallbacks'} of this handle (afmm_tree_counters)."""
        g, f = _ll(), _ll()
        self._check(_lib.afmm_tree_counters(self._h, C.byref(g), C.byref(f)), "afmm_tree_counters")
        return {"graph_launches": g.value, "sort_fallbacks": f.value}

    def copy_out(self, n):
        inf = self.info()
        L, nnz = inf["n_leaves"], inf["nnz"]
        out = {"perm": np.empty(n, np.int32), "leaf_start": np.empty(L, np.int32),
               "leaf_count": np.empty(L, np.int32), "leaf_level": np.empty(L, np.int32),
               "leaf_prefix": np.empty(L, np.uint64), "u_off": np.empty(L + 1, np.int64),
               "u_idx": np.empty(max(nnz, 1), np.int32)}
        self._check(_lib.afmm_tree_copy_out(self._h, *[_ptr(out[k]) for k in
                                                      ("perm", "leaf_start", "leaf_count", "leaf_level",
                                                       "leaf_prefix", "u_off", "u_idx")]),
                    "afmm_tree_copy_out")
        out["u_idx"] = out["u_idx"][:nnz]
        out.update(inf)
        return out

    def farfield_counts(self):
        """M(Op) = [P2M, M2M, M2L, L2L, L2P, P2P] of the last build (L18 SIV.D)."""
        out = np.zeros(6, np.int64)
        self._check(_lib.afmm_tree_farfield_counts(self._h, _ptr(out)), "afmm_tree_farfield_counts")
        return out

    def device_arrays(self):
        """Device pointers (ints) of the last build: perm, leaf_start, leaf_count, u_off, u_idx."""
        ps = [_p() for _ in range(5)]
        self._check(_lib.afmm_tree_device_arrays(self._h, *[C.byref(q) for q in ps]), "afmm_tree_device_arrays")
        return {k: q.value for k, q in zip(("perm", "leaf_start", "leaf_count", "u_off", "u_idx"), ps)}

    def gather(self, src, dst):
        """dst[p] = src[perm[p]] (device tensors)."""
        self._check(_lib.afmm_tree_gather(self._h, _ptr(src), _ptr(dst)), "afmm_tree_gather")

    def gather_rows(self, src, dst):
        """afmm_tree_gather_rows: every row of a contiguous (rows, n) device tensor
        into tree order in one kernel."""
        if src.dim() != 2 or not src.is_contiguous() or not dst.is_contiguous() or dst.shape != src.shape:
            raise ValueError("gather_rows takes two contiguous (rows, n) tensors of the same shape")
        self._check(_lib.afmm_tree_gather_rows(self._h, int(src.shape[0]), _ptr(src), _ptr(dst)),
                    "afmm_tree_gather_rows")

    def scatter(self, src, dst):
        self._check(_lib.afmm_tree_scatter(self._h, _ptr(src), _ptr(dst)), "afmm_tree_scatter")


# ------------------------------------------------------------------ load balancer (row f3)

def lb_predict(counts, coef):
    """afmm_lb_predict (L18 SIV.D): (t_cpu, t_gpu, t) = (sum of the five far-field C_op M(op),
    C_P2P M(P2P), their max) from counts[6] (P2M, M2M, M2L, L2L, L2P, P2P) and coef[6]."""
    m, c = _np(counts, np.int64), _np(coef, np.float64)
    if m.shape != (6,) or c.shape != (6,):
        raise ValueError("counts and coef hold 6 values (P2M, M2M, M2L, L2L, L2P, P2P)")
    tc, tg, t = _d(), _d(), _d()
    st = _lib.afmm_lb_predict(_ptr(m), _ptr(c), C.byref(tc), C.byref(tg), C.byref(t))
    if st:
        raise AfmmError(st, "afmm_lb_predict")
    return tc.value, tg.value, t.value


class LoadBalancer:
    """afmm_lb: the paper's Search / Incremental / Observation controller (L18 SV, L20-L22)."""

    def __init__(self, S_init=128, S_min=8, S_max=2048, dS=8, balance_rel=0.15, observe_rel=0.05):
        cfg = LbConfig()
        _lib.afmm_lb_config_init(C.byref(cfg))
        cfg.S_init, cfg.S_min, cfg.S_max, cfg.dS = int(S_init), int(S_min), int(S_max), int(dS)
        cfg.balance_rel, cfg.observe_rel = float(balance_rel), float(observe_rel)
        h = _p()
        st = _lib.afmm_lb_create(C.byref(cfg), C.byref(h))
        if st:
            raise AfmmError(st, "afmm_lb_create")
        self._h = h

    def step(self, t_cpu, t_gpu):
        a, S = _i(), _i()
        st = _lib.afmm_lb_step(self._h, float(t_cpu), float(t_gpu), C.byref(a), C.byref(S))
        if st:
            raise AfmmError(st, "afmm_lb_step")
        return a.value, S.value

    def predicted(self, t_pred):
        a = _i()
        st = _lib.afmm_lb_predicted(self._h, float(t_pred), C.byref(a))
        if st:
            raise AfmmError(st, "afmm_lb_predicted")
        return a.value

    def state(self):
        s, S, b = _i(), _i(), _d()
        _lib.afmm_lb_state(self._h, C.byref(s), C.byref(S), C.byref(b))
        return {"state": s.value, "S": S.value, "best": b.value}

    def close(self):
        if getattr(self, "_h", None) and _lib is not None:
            _lib.afmm_lb_destroy(self._h)
        self._h = None

    __del__ = close
