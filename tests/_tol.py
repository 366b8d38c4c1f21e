"""Parity tolerance of DESIGN.md reading R16 (from north_star: relative error
<= 1e-5 per body), shared by the GPU parity tests."""
import numpy as np

REL = 1e-5          # per-body relative bound (north_star)
KAPPA = 10.0        # conditioning threshold for the per-body acceleration bound
ABS_A = 1e-6        # bound in units of A_i = sum_j G m_j |d| / r^3 for kappa > 10


def check(gpu, ref, A, rel=REL):
    """gpu: (phi, ax, ay, az) fp32; ref: same in fp64; A: conditioning scale.
    Returns a dict of error statistics; raises AssertionError on violation."""
    phi, ax, ay, az = (np.asarray(v, np.float64) for v in gpu)
    rphi, rax, ray, raz = (np.asarray(v, np.float64) for v in ref)
    # potential: all terms share a sign -> per-body relative error, exact zeros
    zero = rphi == 0
    assert np.array_equal(phi[zero], rphi[zero]), "phi must be exactly 0 where the oracle is 0"
    ephi = np.abs(phi - rphi) / np.where(zero, 1.0, np.abs(rphi))
    assert np.isfinite(ephi).all()
    a = np.stack([ax, ay, az], 1)
    ra = np.stack([rax, ray, raz], 1)
    da = np.linalg.norm(a - ra, axis=1)
    na = np.linalg.norm(ra, axis=1)
    glob = np.linalg.norm(a - ra) / max(np.linalg.norm(ra), 1e-300)
    kappa = np.where(na > 0, A / np.where(na > 0, na, 1.0), np.inf)
    well = kappa <= KAPPA
    ea = np.where(na > 0, da / np.where(na > 0, na, 1.0), 0.0)
    stats = {"phi_max_rel": float(ephi.max()), "a_global_rel": float(glob),
             "a_max_rel_all": float(ea.max()) if ea.size else 0.0,      # strict per-body max
             "a_max_rel_well": float(ea[well].max()) if well.any() else 0.0,
             "a_p999_rel": float(np.quantile(ea, 0.999)), "n_ill": int((~well).sum()),
             "a_max_abs_over_A_ill": float((da[~well] / np.maximum(A[~well], 1e-300)).max()) if (~well).any() else 0.0}
    assert ephi.max() <= rel, stats
    assert glob <= rel, stats
    assert (ea[well] <= rel).all(), stats
    assert (da[~well] <= ABS_A * A[~well] + 1e-300).all(), stats
    return stats


def check_vec(gpu, ref, A, rel=REL):
    """Vector-only version of `check` (Stokeslet velocities): gpu/ref = (ux, uy, uz)."""
    u = np.stack([np.asarray(v, np.float64) for v in gpu], 1)
    r = np.stack([np.asarray(v, np.float64) for v in ref], 1)
    du = np.linalg.norm(u - r, axis=1)
    nr = np.linalg.norm(r, axis=1)
    glob = np.linalg.norm(u - r) / max(np.linalg.norm(r), 1e-300)
    kappa = np.where(nr > 0, A / np.where(nr > 0, nr, 1.0), np.inf)
    well = kappa <= KAPPA
    eu = np.where(nr > 0, du / np.where(nr > 0, nr, 1.0), 0.0)
    stats = {"u_global_rel": float(glob), "u_max_rel_well": float(eu[well].max()) if well.any() else 0.0,
             "n_ill": int((~well).sum())}
    assert np.isfinite(u).all(), stats
    assert glob <= rel, stats
    assert (eu[well] <= rel).all(), stats
    assert (du[~well] <= ABS_A * A[~well] + 1e-300).all(), stats
    return stats
