"""Pins for the oracle's regularized-Stokeslet near field (reading R26; the
paper's second application, L22 SVIII.B / L26 SIX.B; row f4).  Checked against
an independent numpy implementation of the blob-regularized Stokes flow
through its closed forms: the self term, the two-body formula written as a
3x3 matrix, the Oseen (singular Stokeslet) limit far from the blob, the
symmetry of the mobility matrix (reciprocity) and linearity in the forces."""
import numpy as np
import pytest

import oracle
import synth

PI8 = 8 * np.pi


def _S(d, eps2, mu=1.0):
    """Regularized Stokeslet matrix S(d) = [(r^2 + 2e^2) I + d d^T] / (8 pi mu (r^2+e^2)^{3/2})."""
    r2 = float(d @ d)
    return ((r2 + 2 * eps2) * np.eye(3) + np.outer(d, d)) / (PI8 * mu * (r2 + eps2) ** 1.5)


def test_single_body_self_term():
    x = np.array([0.3], np.float32)
    f = np.array([0.5], np.float32), np.array([-0.25], np.float32), np.array([1.0], np.float32)
    T = oracle.Tree(x, x, x, 4)
    ux, uy, uz = oracle.stokeslet(x, x, x, *f, T.leaf_start, T.leaf_count, T.u_off, T.u_idx, 2.0, 1e-4)
    eps = np.sqrt(1e-4)
    for u, fk in zip((ux, uy, uz), f):
        assert u[0] == pytest.approx(float(fk[0]) / (4 * np.pi * 2.0 * eps), rel=1e-14)


def test_two_bodies_matrix_form():
    x = np.array([0.1, 0.7], np.float32)
    y = np.array([0.2, 0.4], np.float32)
    z = np.array([0.9, 0.3], np.float32)
    fx, fy, fz = (np.array(v, np.float32) for v in ([1.0, -0.5], [0.25, 2.0], [-1.5, 0.75]))
    T = oracle.Tree(x, y, z, 4)
    xs, ys, zs, gx, gy, gz = T.sorted_bodies(x, y, z, fx, fy, fz)
    eps2, mu = 1e-2, 1.5
    u = np.stack(oracle.stokeslet(xs, ys, zs, gx, gy, gz, T.leaf_start, T.leaf_count, T.u_off, T.u_idx, mu, eps2), 1)
    P = np.stack([xs, ys, zs], 1).astype(float)
    F = np.stack([gx, gy, gz], 1).astype(float)
    for i in range(2):
        ref = sum(_S(P[i] - P[k], eps2, mu) @ F[k] for k in range(2))
        assert np.allclose(u[i], ref, rtol=1e-13, atol=0)


def test_oseen_limit_far_from_blob():
    """r >> eps: S -> (I/r + d d^T / r^3) / (8 pi mu), relative error O(eps^2/r^2)."""
    x = np.array([0.0, 0.5], np.float32)
    y = np.zeros(2, np.float32)
    z = np.zeros(2, np.float32)
    f = (np.array([0.0, 1.0], np.float32), np.array([0.0, 2.0], np.float32), np.array([0.0, -1.0], np.float32))
    T = oracle.Tree(x, y, z, 4)
    xs, ys, zs, gx, gy, gz = T.sorted_bodies(x, y, z, *f)
    eps2 = 1e-10
    u = np.stack(oracle.stokeslet(xs, ys, zs, gx, gy, gz, T.leaf_start, T.leaf_count, T.u_off, T.u_idx, 1.0, eps2), 1)
    i = int(np.argmin(xs))                 # the force-free body at the origin
    d = np.array([xs[i] - xs[1 - i], 0.0, 0.0])
    r = abs(d[0])
    oseen = (np.eye(3) / r + np.outer(d, d) / r ** 3) / PI8 @ np.array([1.0, 2.0, -1.0])
    assert np.allclose(u[i], oseen, rtol=1e-8)


def test_reciprocity_and_linearity():
    """Symmetric U-lists and S(d) = S(-d)^T = S(d)^T make the near-field mobility
    symmetric: f' . (M f) = f . (M f').  And M(a f + b g) = a M f + b M g."""
    x, y, z, fx, fy, fz = synth.uniform_with_forces(3000, 3)
    _, _, _, gx, gy, gz = synth.uniform_with_forces(3000, 4)
    T = oracle.Tree(x, y, z, 40)
    xs, ys, zs, fx, fy, fz, gx, gy, gz = T.sorted_bodies(x, y, z, fx, fy, fz, gx, gy, gz)
    args = (T.leaf_start, T.leaf_count, T.u_off, T.u_idx, 1.0, 1e-4)
    Mf = np.stack(oracle.stokeslet(xs, ys, zs, fx, fy, fz, *args), 1)
    Mg = np.stack(oracle.stokeslet(xs, ys, zs, gx, gy, gz, *args), 1)
    F = np.stack([fx, fy, fz], 1).astype(float)
    Gm = np.stack([gx, gy, gz], 1).astype(float)
    assert (Gm * Mf).sum() == pytest.approx((F * Mg).sum(), rel=1e-12)
    # linearity with fp32-exact combinations: disjoint supports, and scaling by 2
    even = (np.arange(xs.shape[0]) % 2 == 0)
    fe = [np.where(even, a, 0).astype(np.float32) for a in (fx, fy, fz)]
    go = [np.where(~even, b, 0).astype(np.float32) for b in (gx, gy, gz)]
    h = [(np.float32(2) * a + b).astype(np.float32) for a, b in zip(fe, go)]
    Mfe = np.stack(oracle.stokeslet(xs, ys, zs, *fe, *args), 1)
    Mgo = np.stack(oracle.stokeslet(xs, ys, zs, *go, *args), 1)
    Mh = np.stack(oracle.stokeslet(xs, ys, zs, *h, *args), 1)
    assert np.allclose(Mh, 2 * Mfe + Mgo, rtol=1e-12, atol=1e-12 * np.abs(Mh).max())


def test_single_leaf_equals_dense_sum():
    x, y, z, fx, fy, fz = synth.uniform_with_forces(200, 9)
    T = oracle.Tree(x, y, z, 500)
    args = (T.leaf_start, T.leaf_count, T.u_off, T.u_idx, 0.7, 1e-3)
    xs, ys, zs, gx, gy, gz = T.sorted_bodies(x, y, z, fx, fy, fz)
    u = np.stack(oracle.stokeslet(xs, ys, zs, gx, gy, gz, *args), 1)
    P = np.stack([xs, ys, zs], 1).astype(float)
    F = np.stack([gx, gy, gz], 1).astype(float)
    ref = np.array([sum(_S(P[i] - P[k], 1e-3, 0.7) @ F[k] for k in range(200)) for i in range(200)])
    assert np.allclose(u, ref, rtol=1e-12, atol=1e-12 * np.abs(ref).max())
