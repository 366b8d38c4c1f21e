"""The load-balanced C5 time loop on the GPU (PAPER L18 SV,
L20 SVI-SVII, L22): the controller walks Search -> Incremental -> Observation,
and every tree the loop builds equals the oracle's tree for the controller's
action (KEEP: previous structure; ENFORCE: Enforce_S; REBUILD: fresh build with
the new S), bit-exact, on the GPU's own positions.  FineGrainedOptimize steps
are checked by their contract (valid tree, prediction not worse)."""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

KEYS = ("perm", "leaf_start", "leaf_count", "leaf_level", "leaf_prefix", "u_off", "u_idx")


def _structure(P, nodes, dom):
    """Oracle tree with the GPU tree's structure over positions P (the positions
    that tree was built on): a one-leaf tree, then PushDown of every internal
    node of the GPU tree under the KEEP rule."""
    n = P[0].shape[0]
    base = oracle.Tree(*P, n, domain=dom, ulist=False)
    ed = [(int(l), int(p), 2) for l, p, c in zip(nodes["level"], nodes["prefix"], nodes["nchild"]) if c > 0]
    return base.rebuild(*P, mode=2, edits=ed, ulist=False)


def test_lb_timeloop_trees_and_states():
    import paper_conf_ipps_overmanpmm13_b200 as afmm
    from paper_conf_ipps_overmanpmm13_b200.timeloop import TimeLoop
    n, eps2, dt = 1 << 16, 1e-4, 0.05
    x, y, z, m, vx, vy, vz = synth.colliding_with_velocities(n, 5)
    dom = synth.c5_domain(x, y, z)
    lb = afmm.LoadBalancer(S_init=64, S_min=8, S_max=1024, dS=16)
    loop = TimeLoop(x, y, z, m, vx, vy, vz, 64, eps2, dt, dom, lb=lb, cpu_coef=(2e-9, 4e-9, 4e-9, 4e-9, 2e-9))
    prev = {"P": (x, y, z), "nodes": loop.tree.nodes(), "S": 64}
    seen = {"keep": 0, "rebuild": 0, "enforce": 0, "fine": 0}
    states = []

    def post_maintain(lp, rec):
        P = tuple(lp.state[a].cpu().numpy() for a in range(3))
        G = lp.tree.copy_out(n)
        act = rec["action"]
        seen[act] += 1
        if act == "rebuild":
            want = oracle.Tree(*P, lp.S, domain=dom)
        elif act == "keep":
            want = _structure(prev["P"], prev["nodes"], dom).rebuild(*P, mode=2)
        elif act == "enforce" and "fine" not in rec:
            want = _structure(prev["P"], prev["nodes"], dom).enforce(*P, S=lp.S)
        else:
            want = None
            if "fine" in rec:
                assert rec["fine"]["t_after"] <= rec["fine"]["t_before"]
            assert int(G["leaf_count"].sum()) == n
        if want is not None:
            for k in KEYS:
                assert np.array_equal(G[k], getattr(want, k)), (lp.step_no, act, k)
        prev.update(P=P, nodes=lp.tree.nodes(), S=lp.S)

    for _ in range(40):
        rec = loop.step({"post_maintain": post_maintain})
        states.append(rec["lb_state"])
        assert 8 <= rec["S_next"] <= 1024
        assert rec["t_gpu"] > 0 and rec["t_cpu_model"] > 0
    assert states[0] == afmm.LB_SEARCH or states[0] == afmm.LB_INCREMENTAL
    assert afmm.LB_OBSERVATION in states                       # the controller settles
    assert seen["rebuild"] >= 2 and seen["keep"] >= 5
    loop.close()
