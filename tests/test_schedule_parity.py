"""viper_schedule (C++, libviper.so) against the schedule oracle
(oracle/sched_ref.py).  Host-only: runs without a GPU."""
import math

import numpy as np
import pytest

from oracle import sched_ref as S
from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V


def _curve(kind, rng, n):
    x = np.arange(n, dtype=np.float64)
    if kind == "exp3":
        y = rng.uniform(1, 3) * np.exp(-rng.uniform(0.02, 0.2) * x) + rng.uniform(0.05, 0.5)
    elif kind == "exp2":
        y = rng.uniform(1, 3) * np.exp(-rng.uniform(0.02, 0.2) * x)
    else:
        y = rng.uniform(1, 3) - rng.uniform(0.001, 0.02) * x
    return x, y + rng.normal(0, 0.005, n)


@pytest.mark.parametrize("case", range(24))
def test_fit_parity(case):
    rng = np.random.default_rng(case)
    kind = ["exp3", "exp2", "lin"][case % 3]
    x, y = _curve(kind, rng, int(rng.integers(20, 80)))
    fam, p, mses = S.fit_tlp(x, y)
    out = V.schedule(list(y), s_iter=0, e_iter=10, total_infers=100, t_train=1.0, t_infer=1.0, t_p=0.0,
                     t_c=0.0, x=list(x))
    for f in range(4):
        # both sides are local least-squares optimisers: the C++ fit must be at
        # least as good as scipy's (equal on well-posed families)
        assert out["mse"][f] <= mses[f] * (1 + 1e-6) + 1e-15, (f, out["mse"], mses)
        if kind == "exp3" and f in (S.EXP3, S.EXPD3) or kind == "exp2" and f == S.EXP2 or f == S.LIN2:
            assert out["mse"][f] == pytest.approx(mses[f], rel=1e-6, abs=1e-15)
    srt = sorted(out["mse"])
    if abs(srt[0] - srt[1]) > 1e-3 * srt[1]:  # a clear winner: both pick it
        assert out["family"] == fam
        assert out["params"][: S.NPARAMS[fam]] == pytest.approx(list(p[: S.NPARAMS[fam]]), rel=1e-4, abs=1e-7)


@pytest.mark.parametrize("case", range(30))
def test_algorithms_exact_given_params(case):
    rng = np.random.default_rng(1000 + case)
    fam = int(rng.integers(0, 4))
    params = [float(rng.uniform(0.5, 3)), float(rng.uniform(0.01, 0.2)), float(rng.uniform(0.05, 0.6))]
    if fam == S.LIN2:
        params = [-float(rng.uniform(0.001, 0.05)), float(rng.uniform(1, 3)), 0.0]
    tt, ti = float(rng.uniform(0.02, 0.2)), float(rng.uniform(0.002, 0.02))
    tp, tc = float(rng.uniform(0, 0.5)), float(rng.uniform(0, 0.5))
    s = int(rng.integers(0, 20))
    e = s + int(rng.integers(1, 120))
    M = int(rng.integers(10, 50000))
    L = lambda it: float(S.predict(fam, params, it))
    bi, ml = S.fixed_interval(L, s, e, M, tt, tp, tc, ti)
    out = V.schedule(None, s_iter=s, e_iter=e, total_infers=M, t_train=tt, t_infer=ti, t_p=tp, t_c=tc,
                     family=fam, params=params)
    assert out["best_interval"] == bi
    assert out["predicted_cil"] == pytest.approx(ml, rel=1e-12)
    th = float(rng.uniform(0.0005, 0.05))
    sc, pc = S.greedy(L, s, e, M, th, tt, tp, tc, ti)
    g = V.schedule(None, s_iter=s, e_iter=e, total_infers=M, t_train=tt, t_infer=ti, t_p=tp, t_c=tc,
                   family=fam, params=params, algo=V.SCHED_GREEDY, thresh=th)
    assert g["sched"] == sc
    assert g["predicted_cil"] == pytest.approx(pc, rel=1e-12)


def test_worked_example_end_to_end():
    x = np.arange(30.0)
    y = 2.0 * np.exp(-0.05 * x) + 0.3
    ref = S.schedule(y, 0, 40, 500, 7.0, 1.0, s_model=3e9, bw_write=1e9, bw_read=1.5e9)
    out = V.schedule(list(y), s_iter=0, e_iter=40, total_infers=500, t_train=7.0, t_infer=1.0, s_model=3e9,
                     bw_write=1e9, bw_read=1.5e9)
    assert out["family"] == ref["family"] == S.EXP3
    assert out["params"] == pytest.approx(list(ref["params"]), rel=1e-7)
    assert out["best_interval"] == ref["best_interval"] == 4
    assert out["sched"] == ref["sched"]
    assert out["predicted_cil"] == pytest.approx(500.629627, abs=1e-5)


def test_greedy_threshold_from_warmup():
    rng = np.random.default_rng(3)
    y = 2.0 * np.exp(-0.05 * np.arange(40)) + 0.3 + rng.normal(0, 0.003, 40)
    ref = S.schedule(y, 0, 200, 5000, 0.1, 0.01, t_p=0.05, t_c=0.02, algo=1)
    out = V.schedule(list(y), s_iter=0, e_iter=200, total_infers=5000, t_train=0.1, t_infer=0.01, t_p=0.05,
                     t_c=0.02, algo=V.SCHED_GREEDY)
    assert out["thresh"] == pytest.approx(ref["thresh"], rel=1e-12)
    if out["family"] == ref["family"]:
        assert out["sched"] == ref["sched"]


def test_size_query_protocol():
    import ctypes as C
    L = V.lib()
    la = (C.c_double * 3)(1.0, 0.8, 0.7)
    si = V.viper_sched_in(la, None, 3, 0, 10, 100, 1.0, 1.0, 0.0, 0.0, 0.0, 0.0, 0.0, 0, -1.0, 1,
                          (C.c_double * 3)(1.0, 0.1, 0.0))
    so = V.viper_sched_out()
    so.sched_cap = 0
    assert L.viper_schedule(C.byref(si), C.byref(so)) == V.E_INVAL
    assert so.sched_len == 10 // so.best_interval


def test_bad_inputs():
    with pytest.raises(V.ViperError):
        V.schedule([1.0, 0.5], s_iter=0, e_iter=5, total_infers=10, t_train=1.0, t_infer=1.0, t_p=0.0, t_c=0.0)
    with pytest.raises(V.ViperError):
        V.schedule([1.0, 0.9, 0.8], s_iter=5, e_iter=0, total_infers=10, t_train=1.0, t_infer=1.0, t_p=0, t_c=0)
