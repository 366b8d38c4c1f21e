"""fp64 CPU oracle for the AFMM near-field P2P path -- TEST INFRASTRUCTURE.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` legs may import this package.  The product path
(``paper_conf_ipps_overmanpmm13_b200``) never imports it and shares no code with
it.  The arithmetic lives in ``oracle.c`` (plain C,
``-ffp-contract=off``); this module only marshals numpy arrays through ctypes.

Every function cites the passage of /root/reference/PAPER.md it follows; see
oracle.c's header.  Pins: tests/test_oracle.py.  Parity unpinned: none.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile oracle.c -> liboracle.so (gcc, -O2 -fopenmp -ffp-contract=off)."""
    src = os.path.join(_HERE, "oracle.c")
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-ffp-contract=off", "-fno-fast-math",
                               "-fPIC", "-shared", "-std=c11", "-o", _LIB_PATH, src, "-lm"])
    return _LIB_PATH


def _L():
    global _lib
    if _lib is None:
        build()
        lib = C.CDLL(_LIB_PATH)
        p = C.c_void_p
        i64 = C.c_int64
        lib.oracle_tree_build.restype = p
        lib.oracle_tree_build.argtypes = [i64, p, p, p, C.c_int, C.c_int, p, C.c_int]
        lib.oracle_tree_nleaves.restype = i64
        lib.oracle_tree_nleaves.argtypes = [p]
        lib.oracle_tree_nnodes.restype = i64
        lib.oracle_tree_nnodes.argtypes = [p]
        lib.oracle_tree_get.restype = None
        lib.oracle_tree_get.argtypes = [p] * 8
        lib.oracle_tree_nodes.restype = None
        lib.oracle_tree_nodes.argtypes = [p] * 6
        lib.oracle_ulist_build.restype = i64
        lib.oracle_ulist_build.argtypes = [p]
        lib.oracle_ulist_get.restype = None
        lib.oracle_ulist_get.argtypes = [p, p, p]
        lib.oracle_tree_free.restype = None
        lib.oracle_tree_free.argtypes = [p]
        lib.oracle_domain.restype = None
        lib.oracle_domain.argtypes = [i64, p, p, p, p, p]
        lib.oracle_p2p.restype = None
        lib.oracle_p2p.argtypes = [i64, p, p, p, p, i64, p, p, p, p, C.c_double, C.c_double,
                                   i64, p, p, p, p, p, p]
        lib.oracle_interactions.restype = None
        lib.oracle_interactions.argtypes = [i64, p, p, p, p]
        lib.oracle_tree_enforce.restype = p
        lib.oracle_tree_enforce.argtypes = [p, i64, p, p, p, C.c_int]
        lib.oracle_tree_rebuild.restype = p
        lib.oracle_tree_rebuild.argtypes = [p, i64, p, p, p, C.c_int, C.c_int, i64, p, p, p]
        lib.oracle_kick.restype = None
        lib.oracle_kick.argtypes = [i64, p, p, p, p, p, p, C.c_double]
        lib.oracle_drift.restype = None
        lib.oracle_drift.argtypes = [i64, p, p, p, p, p, p, C.c_double]
        lib.oracle_stokeslet.restype = None
        lib.oracle_stokeslet.argtypes = [i64, p, p, p, p, p, p, i64, p, p, p, p, C.c_double, C.c_double,
                                         i64, p, p, p, p, p]
        lib.oracle_farfield_counts.restype = None
        lib.oracle_farfield_counts.argtypes = [p, p]
        lib.oracle_partition_literal.restype = None
        lib.oracle_partition_literal.argtypes = [i64, p, C.c_int, p, p]
        _lib = lib
    return _lib


def _ptr(a):
    return None if a is None else a.ctypes.data_as(C.c_void_p)


def _c(a, dt):
    return np.ascontiguousarray(a, dtype=dt)


class Tree:
    """Adaptive octree + U-list of the oracle (fields are numpy copies).

    Keeps its C handle so that ``enforce`` (Enforce_S, L20 SVI.A) can walk it."""

    def __init__(self, x=None, y=None, z=None, S=None, domain=None, ulist=True, _handle=None, _n=None):
        lib = _L()
        if _handle is None:
            x, y, z = (_c(v, np.float32) for v in (x, y, z))
            n = x.shape[0]
            lo = np.zeros(3)
            k = 0
            fixed = 0
            if domain is not None:
                lo = _c(domain[0], np.float64)
                k = int(domain[1])
                fixed = 1
            h = lib.oracle_tree_build(n, _ptr(x), _ptr(y), _ptr(z), int(S), fixed, _ptr(lo), k)
            if not h:
                raise ValueError("oracle_tree_build failed")
        else:
            h, n = _handle, _n
        self._h = h
        self._fill(lib, h, n, int(S), ulist)

    def _fill(self, lib, h, n, S, ulist):
        L = lib.oracle_tree_nleaves(h)
        self.n, self.S, self.L = n, S, int(L)
        self.perm = np.empty(n, np.int32)
        self.leaf_start = np.empty(L, np.int32)
        self.leaf_count = np.empty(L, np.int32)
        self.leaf_level = np.empty(L, np.int32)
        self.leaf_prefix = np.empty(L, np.uint64)
        lo_out = np.empty(3)
        k_out = np.zeros(1, np.int32)
        lib.oracle_tree_get(h, _ptr(self.perm), _ptr(self.leaf_start), _ptr(self.leaf_count),
                            _ptr(self.leaf_level), _ptr(self.leaf_prefix), _ptr(lo_out), _ptr(k_out))
        self.lo, self.k = lo_out, int(k_out[0])
        nn = lib.oracle_tree_nnodes(h)
        self.node_level = np.empty(nn, np.int32)
        self.node_prefix = np.empty(nn, np.uint64)
        self.node_b = np.empty(nn, np.int64)
        self.node_e = np.empty(nn, np.int64)
        self.node_is_leaf = np.empty(nn, np.int32)
        lib.oracle_tree_nodes(h, _ptr(self.node_level), _ptr(self.node_prefix), _ptr(self.node_b),
                              _ptr(self.node_e), _ptr(self.node_is_leaf))
        if ulist:
            nnz = lib.oracle_ulist_build(h)
            self.u_off = np.empty(L + 1, np.int64)
            self.u_idx = np.empty(max(nnz, 1), np.int32)
            lib.oracle_ulist_get(h, _ptr(self.u_off), _ptr(self.u_idx))
            self.u_idx = self.u_idx[:nnz]

    def enforce(self, x, y, z, S=None, ulist=True):
        """Enforce_S (L20 SVI.A) for new positions of the same bodies -> new Tree.
        x, y, z are given in THIS tree's body order (positions after a drift)."""
        x, y, z = (_c(v, np.float32) for v in (x, y, z))
        S = self.S if S is None else int(S)
        h = _L().oracle_tree_enforce(self._h, x.shape[0], _ptr(x), _ptr(y), _ptr(z), S)
        if not h:
            raise ValueError("oracle_tree_enforce failed")
        return Tree(S=S, ulist=ulist, _handle=h, _n=x.shape[0])

    def rebuild(self, x, y, z, S=None, mode=2, edits=(), ulist=True):
        """Rebuild for new positions with the previous structure (mode 2, KEEP)
        or the Enforce_S rule (mode 1), then Collapse (1) / PushDown (2) edits
        given as (level, prefix, action) triples (L18 SIV.B-C, L20 SVI.B; R27)."""
        x, y, z = (_c(v, np.float32) for v in (x, y, z))
        S = self.S if S is None else int(S)
        lev = _c([e[0] for e in edits] or [0], np.int32)
        pre = _c([e[1] for e in edits] or [0], np.uint64)
        act = _c([e[2] for e in edits] or [0], np.int32)
        h = _L().oracle_tree_rebuild(self._h, x.shape[0], _ptr(x), _ptr(y), _ptr(z), S, int(mode),
                                     len(edits), _ptr(lev), _ptr(pre), _ptr(act))
        if not h:
            raise ValueError("oracle_tree_rebuild failed")
        return Tree(S=S, ulist=ulist, _handle=h, _n=x.shape[0])

    def farfield_counts(self):
        """M(Op) for P2M, M2M, M2L, L2L, L2P, P2P (L18 SIV.D; reading R27)."""
        out = np.zeros(6, np.int64)
        _L().oracle_farfield_counts(self._h, _ptr(out))
        return out

    def __del__(self):
        if getattr(self, "_h", None) and _lib is not None:
            _lib.oracle_tree_free(self._h)
            self._h = None

    def sorted_bodies(self, *arrs):
        """Permute input-order arrays into tree (Morton) order."""
        return tuple(_c(a, np.float32)[self.perm] for a in arrs)


def set_threads(n: int) -> None:
    """OpenMP threads of the oracle's parallel loops (omp_set_num_threads of the
    libgomp the oracle links; e.g. 1 for a one-core baseline).  No arithmetic."""
    _L().omp_set_num_threads(int(n))


def kick(vx, vy, vz, ax, ay, az, h):
    """Leapfrog kick v <- v + h a (fp64 arithmetic on fp32 state, one rounding)."""
    v = [np.array(a, np.float32) for a in (vx, vy, vz)]
    a = [_c(t, np.float32) for t in (ax, ay, az)]
    _L().oracle_kick(v[0].shape[0], *[_ptr(t) for t in v], *[_ptr(t) for t in a], float(h))
    return tuple(v)


def drift(x, y, z, vx, vy, vz, dt):
    """Leapfrog drift x <- x + dt v (fp64 arithmetic on fp32 state, one rounding)."""
    p = [np.array(a, np.float32) for a in (x, y, z)]
    v = [_c(t, np.float32) for t in (vx, vy, vz)]
    _L().oracle_drift(p[0].shape[0], *[_ptr(t) for t in p], *[_ptr(t) for t in v], float(dt))
    return tuple(p)


def domain(x, y, z):
    x, y, z = (_c(v, np.float32) for v in (x, y, z))
    lo = np.empty(3)
    k = np.zeros(1, np.int32)
    _L().oracle_domain(x.shape[0], _ptr(x), _ptr(y), _ptr(z), _ptr(lo), _ptr(k))
    return lo, int(k[0])


def p2p(x, y, z, m, leaf_start, leaf_count, u_off, u_idx, G=1.0, eps2=0.0, targets=None,
        with_scale=False):
    """fp64 naive P2P over bodies in tree order.  Returns (phi, ax, ay, az[, A]).

    If ``targets`` (leaf ids) is given only those leaves' bodies are computed;
    other entries are NaN."""
    x, y, z, m = (_c(v, np.float32) for v in (x, y, z, m))
    leaf_start, leaf_count = _c(leaf_start, np.int32), _c(leaf_count, np.int32)
    u_off, u_idx = _c(u_off, np.int64), _c(u_idx, np.int32)
    n = x.shape[0]
    L = leaf_start.shape[0]
    out = [np.full(n, np.nan) for _ in range(5 if with_scale else 4)]
    tg = None if targets is None else _c(targets, np.int32)
    _L().oracle_p2p(n, _ptr(x), _ptr(y), _ptr(z), _ptr(m), L, _ptr(leaf_start),
                    _ptr(leaf_count), _ptr(u_off), _ptr(u_idx), float(G), float(eps2),
                    0 if tg is None else tg.shape[0], _ptr(tg),
                    *[_ptr(o) for o in out[:4]], _ptr(out[4]) if with_scale else None)
    return tuple(out)


def stokeslet(x, y, z, fx, fy, fz, leaf_start, leaf_count, u_off, u_idx, mu=1.0, eps2=1e-6,
              targets=None, with_scale=False):
    """fp64 regularized-Stokeslet near field (reading R26) over bodies in tree
    order; self term included.  Returns (ux, uy, uz[, A])."""
    arrs = [_c(v, np.float32) for v in (x, y, z, fx, fy, fz)]
    leaf_start, leaf_count = _c(leaf_start, np.int32), _c(leaf_count, np.int32)
    u_off, u_idx = _c(u_off, np.int64), _c(u_idx, np.int32)
    n = arrs[0].shape[0]
    out = [np.full(n, np.nan) for _ in range(4 if with_scale else 3)]
    tg = None if targets is None else _c(targets, np.int32)
    _L().oracle_stokeslet(n, *[_ptr(a) for a in arrs], leaf_start.shape[0], _ptr(leaf_start), _ptr(leaf_count),
                          _ptr(u_off), _ptr(u_idx), float(mu), float(eps2), 0 if tg is None else tg.shape[0],
                          _ptr(tg), *[_ptr(o) for o in out[:3]], _ptr(out[3]) if with_scale else None)
    return tuple(out)


def interactions(leaf_count, u_off, u_idx):
    leaf_count = _c(leaf_count, np.int32)
    u_off, u_idx = _c(u_off, np.int64), _c(u_idx, np.int32)
    L = leaf_count.shape[0]
    I = np.empty(L, np.int64)
    _L().oracle_interactions(L, _ptr(leaf_count), _ptr(u_off), _ptr(u_idx), _ptr(I))
    return I


def partition_literal(I, G):
    I = _c(I, np.int64)
    L = I.shape[0]
    owner = np.empty(L, np.int32)
    split = np.empty(G + 1, np.int64)
    _L().oracle_partition_literal(L, _ptr(I), int(G), _ptr(owner), _ptr(split))
    return owner, split
