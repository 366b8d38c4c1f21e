"""CPU tests of the C-ABI library: it loads, exports every symbol the headers
declare, and its host-only functions agree with the oracle bit-exactly."""
import ctypes
import os
import re

import numpy as np
import pytest

import oracle
import synth

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    names = []
    for h in ("afmm_p2p.h", "afmm_tree.h", "afmm_step.h", "afmm_balance.h"):
        src = open(os.path.join(ROOT, "include", h)).read()
        src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
        names += re.findall(r"\b(afmm_\w+)\s*\(", src)
    return sorted(set(names))


def test_library_loads_and_exports_every_declared_symbol():
    import paper_conf_ipps_overmanpmm13_b200 as afmm
    lib = ctypes.CDLL(afmm.LIB_PATH)
    decl = _declared()
    assert len(decl) >= 25
    for name in decl:
        assert hasattr(lib, name), name
    assert sorted(afmm.EXPORTED) == decl
    assert "sm_100a" in afmm.version()


def test_library_is_sm100a_cubin():
    import subprocess
    import paper_conf_ipps_overmanpmm13_b200 as afmm
    out = subprocess.run(["cuobjdump", "-lelf", afmm.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


@pytest.mark.parametrize("dist,n,S", [("uniform", 4096, 64), ("plummer", 30000, 32),
                                      ("colliding", 30000, 100)])
def test_interactions_and_literal_partition_bit_exact(dist, n, S):
    import paper_conf_ipps_overmanpmm13_b200 as afmm
    x, y, z, m = synth.make(dist, n, 5)
    T = oracle.Tree(x, y, z, S)
    I_ref = oracle.interactions(T.leaf_count, T.u_off, T.u_idx)
    I = afmm.interactions(T.leaf_count, T.u_off, T.u_idx)
    assert np.array_equal(I, I_ref)
    for G in (1, 2, 3, 4, 8, 16):
        _, split_ref = oracle.partition_literal(I_ref, G)
        assert np.array_equal(afmm.partition_literal(I, G), split_ref)
        # the weighted rule with integer-valued weights gives the same cut
        assert np.array_equal(afmm.partition_weighted(I.astype(np.float64), G), split_ref)


def test_partition_edge_cases():
    import paper_conf_ipps_overmanpmm13_b200 as afmm
    assert list(afmm.partition_literal(np.array([5, 1, 1]), 8)) == [0, 1, 2, 3, 3, 3, 3, 3, 3]
    assert list(afmm.partition_literal(np.array([7]), 1)) == [0, 1]
    assert list(afmm.partition_literal(np.array([1, 1, 1, 1]), 2)) == [0, 2, 4]
    with pytest.raises(afmm.AfmmError):
        afmm.partition_literal(np.array([1, -1]), 2)
    with pytest.raises(afmm.AfmmError):
        afmm.partition_weighted(np.array([1.0, np.nan]), 2)


def test_interactions_rejects_bad_index():
    import paper_conf_ipps_overmanpmm13_b200 as afmm
    with pytest.raises(afmm.AfmmError):
        afmm.interactions(np.array([1, 1]), np.array([0, 1, 2]), np.array([0, 2]))
