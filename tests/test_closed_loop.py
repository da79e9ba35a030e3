"""N2 closed loop (paper_conf_icpp_yecrbypnmskn24_b200/closed_loop.py).

CPU: its CIL accounting on Alg. 1's ideal timeline equals the schedule
oracle's Alg. 2 / Alg. 3 values, with times that are integer
multiples of t_infer, so the reading R11 tie rule is exercised.
GPU: a short closed loop on the C1 workload.  Served versions are monotone
and were all published.  The never-update policy serves exactly L(s_iter).
The IPP schedule's measured CIL is no worse than never updating.
"""
import math

import pytest

from oracle import sched_ref as S
from paper_conf_icpp_yecrbypnmskn24_b200 import closed_loop as CL


def _L(x):
    return 2.0 * math.exp(-0.05 * x) + 0.3


def _alg2_for(i, s, e, total, tt, tp, tc, ti):
    t_l, rem, p_l, c_iter, ver = 0.0, total, _L(s), s + i, 1
    while c_iter <= e:
        il, inf = S.cil(i, p_l, ver, rem, tt, tp, tc, ti)
        t_l, rem = t_l + il, rem - inf
        p_l = _L(c_iter)
        c_iter, ver = c_iter + i, ver + 1
    return t_l + p_l * rem


@pytest.mark.parametrize("s,e,tt,tp,tc,ti,total", [(0, 40, 7.0, 3.0, 2.0, 1.0, 500), (5, 60, 3.0, 2.0, 1.0, 1.0, 300),
                                                   (0, 30, 2.0, 0.0, 0.0, 1.0, 90), (0, 25, 4.0, 6.0, 2.0, 2.0, 80)])
def test_ideal_timeline_equals_alg2(s, e, tt, tp, tc, ti, total):
    for i in range(1, e - s + 1):
        sched = list(range(s + i, e + 1, i))
        got = CL.cil_from_arrivals(_L(s), CL.ideal_arrivals(sched, s, tt, tp, tc, _L), total, ti)
        assert got == pytest.approx(_alg2_for(i, s, e, total, tt, tp, tc, ti), rel=1e-12), i
    bi, ml = S.fixed_interval(_L, s, e, total, tt, tp, tc, ti)
    sims = [CL.cil_from_arrivals(_L(s), CL.ideal_arrivals(list(range(s + i, e + 1, i)), s, tt, tp, tc, _L), total, ti)
            for i in range(1, e - s + 1)]
    assert min(sims) == pytest.approx(ml, rel=1e-12)


def test_ideal_timeline_equals_alg3():
    tt, tp, tc, ti, total = 3.0, 2.0, 1.0, 1.0, 400
    for thresh in (0.2, 0.1, 0.05):
        sc, pc = S.greedy(_L, 0, 60, total, thresh, tt, tp, tc, ti)
        got = CL.cil_from_arrivals(_L(0), CL.ideal_arrivals(sc, 0, tt, tp, tc, _L), total, ti)
        assert got == pytest.approx(pc, rel=1e-12)


def test_no_arrivals_is_initial_loss():
    assert CL.cil_from_arrivals(0.75, [], 123, 0.5) == pytest.approx(0.75 * 123)
    # an arrival exactly at an inference's issue time serves it (R11)
    assert CL.cil_from_arrivals(1.0, [(2.0, 0.0)], 4, 1.0) == pytest.approx(2.0)


@pytest.mark.gpu
def test_closed_loop_c1():
    from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V
    curve = CL.LossCurve(a=2.0, b=0.02, c=0.5, noise=0.0)
    r = CL.run(model="ptychonn", tier=V.TIER_GPU, mode=V.ASYNC, t_train=1e-3, t_infer=5e-4, s_iter=20,
               e_iter=220, fixed=(1, 50), curve=curve, greedy=True, true_best=False)
    pol = r["policies"]
    for name, p in pol.items():
        assert p["versions_monotone_and_published"], name
        assert 0.9 * p["n_publish"] <= p["n_installed"] <= p["n_publish"], name
    never = pol["never"]
    assert never["served_cil"] == pytest.approx(curve(20) * r["total_infers"], rel=1e-12)
    assert never["timeline_cil"] == pytest.approx(never["served_cil"], rel=1e-12)
    ipp = [p for n, p in pol.items() if n.startswith("ipp_fixed")][0]
    assert ipp["timeline_cil"] < never["timeline_cil"]
    assert ipp["served_cil"] < never["served_cil"]
    assert r["schedule"]["family"] in ("Exp3", "Expd3")
