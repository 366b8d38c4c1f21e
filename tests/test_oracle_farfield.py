"""Pins for the oracle's far-field operation counts M(Op) (L18 SIV.D time
prediction; reading R27, CGR V-lists): closed forms on complete trees and
independent brute force on adaptive ones."""
import numpy as np

import oracle
import synth


def _vlist_closed_form(L):
    """Complete octree of depth L on a 2^L grid: |V(b)| for a level-l node at
    cell i (per axis) = prod A_a - prod B_a with A_a = #{c : |c//2 - i//2| <= 1},
    B_a = #{c : |c - i| <= 1}, c in [0, 2^l)."""
    tot = 0
    for lev in range(2, L + 1):
        M = 2 ** lev
        c = np.arange(M)
        A = np.array([np.sum(np.abs(c // 2 - i // 2) <= 1) for i in range(M)])
        B = np.array([np.sum(np.abs(c - i) <= 1) for i in range(M)])
        tot += int((A[:, None, None] * A[None, :, None] * A[None, None, :]).sum()
                   - (B[:, None, None] * B[None, :, None] * B[None, None, :]).sum())
    return tot


def test_counts_complete_tree_closed_form():
    for M in (4, 8):
        x, y, z, m = synth.lattice(M)
        T = oracle.Tree(x, y, z, 1)
        L = int(np.log2(M))
        c = T.farfield_counts()
        nodes = sum(8 ** l for l in range(L + 1))
        assert c[0] == M ** 3 and c[4] == M ** 3                  # P2M, L2P per leaf
        assert c[1] == nodes - 1 and c[3] == nodes - 1            # M2M, L2L per non-root node
        assert c[2] == _vlist_closed_form(L)                       # M2L
        assert c[5] == (3 * M - 2) ** 3                            # P2P pairs of the unit-count leaves
    # interior node of a deep complete tree: |V| = 6^3 - 3^3 = 189
    assert _vlist_closed_form(3) > 0


def test_counts_adaptive_bruteforce():
    """V-list sizes vs an independent brute force over node boxes."""
    x, y, z, m = synth.make("plummer", 3000, 3)
    T = oracle.Tree(x, y, z, 8)
    c = T.farfield_counts()
    lvl = T.node_level.astype(np.int64)
    pre = T.node_prefix.astype(np.uint64)
    q = np.zeros((lvl.size, 3), np.int64)
    for b in range(int(lvl.max())):
        for a in range(3):
            q[:, a] |= np.where(lvl > b, ((pre >> np.uint64(3 * b + a)) & np.uint64(1)).astype(np.int64) << b, 0)
    w = np.int64(1) << (21 - lvl)
    A = q * w[:, None]
    internal = T.node_is_leaf == 0
    key = {(int(l), int(p)): i for i, (l, p) in enumerate(zip(lvl, pre))}

    def touch(i, j):
        return all(A[i, a] <= A[j, a] + w[j] and A[j, a] <= A[i, a] + w[i] for a in range(3))

    m2l = 0
    for b in range(lvl.size):
        if lvl[b] < 2:
            continue
        par = key[(int(lvl[b]) - 1, int(pre[b]) >> 3)]
        for qn in np.nonzero((lvl == lvl[par]) & internal)[0]:
            if not touch(par, qn):
                continue
            for o in range(8):
                ch = key.get((int(lvl[qn]) + 1, (int(pre[qn]) << 3) | o))
                if ch is not None and not touch(b, ch):
                    m2l += 1
    assert c[2] == m2l
    assert c[0] == T.L and c[1] == lvl.size - 1
    I = oracle.interactions(T.leaf_count, T.u_off, T.u_idx)
    assert c[5] == I.sum()
