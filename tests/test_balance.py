"""The load-balancing state machine (row f3; PAPER L18 SV, L20 SVI-SVII, L22),
host-only: driven by a synthetic cost model T_cpu(S) = a/S + b (far field
shrinks as leaves grow) and T_gpu(S) = c S (near field grows), L14 SIII.A Fig. 3."""
import pytest

import paper_conf_ipps_overmanpmm13_b200 as afmm

LB = afmm


def model(S, a=2.0, b=0.01, c=0.0004):
    return a / S + b, c * S


def test_search_then_incremental_then_observation():
    lb = afmm.LoadBalancer(S_init=16, S_min=8, S_max=2048, dS=4, balance_rel=0.15, observe_rel=0.05)
    S = 16
    trace = []
    for _ in range(60):
        cpu, gpu = model(S)
        act, S2 = lb.step(cpu, gpu)
        st = lb.state()
        trace.append((st["state"], act, S2))
        if act == LB.LB_FINE:
            lb.predicted(max(model(S2)))
        S = S2
        if st["state"] == LB.LB_OBSERVATION and act == LB.LB_KEEP:
            break
    states = [t[0] for t in trace]
    # Search first (binary search, a rebuild every step), < 15 steps (L20 SVII.B)
    n_search = states.index(LB.LB_INCREMENTAL) if LB.LB_INCREMENTAL in states else states.index(LB.LB_OBSERVATION)
    assert 0 < n_search < 15
    assert all(t[1] == LB.LB_REBUILD for t in trace[:n_search - 1])
    # ends in Observation near the balance point S* = sqrt(a/c) ~ 70.7
    assert states[-1] == LB.LB_OBSERVATION
    cpu, gpu = model(S)
    assert abs(cpu - gpu) <= 0.3 * max(cpu, gpu)
    assert 50 <= S <= 100


def test_observation_5_percent_rule_enforce_and_fine():
    lb = afmm.LoadBalancer(S_init=64, S_min=8, S_max=2048, dS=4)
    # reach observation quickly: balanced times
    act, S = lb.step(1.0, 1.0)                  # Search: balanced -> Incremental (first step)
    for _ in range(200):
        st = lb.state()
        if st["state"] == LB.LB_OBSERVATION:
            break
        a, S = lb.step(1.0 + 0.001 * (64 - S), 1.0 - 0.001 * (64 - S))
        if a == LB.LB_FINE:
            lb.predicted(1.0)
    assert lb.state()["state"] == LB.LB_OBSERVATION
    best = lb.state()["best"]
    # within 5 %: nothing happens, best tracks the minimum
    assert lb.step(best * 1.04, best * 0.5)[0] == LB.LB_KEEP
    # more than 5 %: Enforce_S ...
    act, _ = lb.step(best * 1.2, best * 0.5)
    assert act == LB.LB_ENFORCE
    with pytest.raises(afmm.AfmmError):                 # a prediction is pending
        lb.step(1.0, 1.0)
    # ... predicted good -> keep; the next step's time becomes the best
    assert lb.predicted(best * 1.01) == LB.LB_KEEP
    assert lb.step(best * 1.3, 0.1)[0] == LB.LB_KEEP
    assert lb.state()["best"] == pytest.approx(best * 1.3)
    best = lb.state()["best"]
    # deviation -> Enforce_S -> predicted bad -> FineGrainedOptimize -> predicted bad -> Incremental next step
    assert lb.step(best * 1.5, 0.1)[0] == LB.LB_ENFORCE
    assert lb.predicted(best * 1.4) == LB.LB_FINE
    assert lb.predicted(best * 1.3) == LB.LB_KEEP
    act, S2 = lb.step(best * 1.5, 0.1)
    assert lb.state()["state"] == LB.LB_INCREMENTAL and act == LB.LB_REBUILD and S2 > S - 100
    with pytest.raises(afmm.AfmmError):
        lb.predicted(1.0)                                # nothing pending


def test_incremental_direction_follows_dominant_unit():
    lb = afmm.LoadBalancer(S_init=100, S_min=8, S_max=2048, dS=10, balance_rel=0.5)
    # balanced within 50 % -> Incremental on the first step; CPU dominates -> S increases
    act, S = lb.step(1.2, 1.0)
    assert lb.state()["state"] == LB.LB_INCREMENTAL and act == LB.LB_REBUILD and S == 110
    act, S = lb.step(1.1, 1.05)
    assert S == 120
    # the GPU becomes dominant: transitional S found, balanced -> Observation
    act, S = lb.step(1.0, 1.1)
    assert lb.state()["state"] == LB.LB_OBSERVATION and act == LB.LB_KEEP and S == 120


def test_invalid_configs():
    for kw in ({"S_init": 4, "S_min": 8}, {"dS": 0}, {"balance_rel": 0.0}, {"S_max": 100, "S_init": 200}):
        with pytest.raises(afmm.AfmmError):
            afmm.LoadBalancer(**kw)
    lb = afmm.LoadBalancer()
    with pytest.raises(afmm.AfmmError):
        lb.step(float("nan"), 1.0)
