"""Pins for the schedule oracle (oracle/sched_ref.py), CPU only.

Pinned against: closed forms of Eq. 2, an independent
discrete-event simulation of the producer/consumer timeline of Fig. 1 /
Alg. 1, special cases of Alg. 2, the survey's
derived worked examples (tests/golden/sched_worked_examples.json) and
library routines for the TLP fits (numpy.polyfit, noise-free recovery).
"""
import json
import math
import os
import statistics

import numpy as np
import pytest

from oracle import sched_ref as S

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "sched_worked_examples.json")))


def _L(a=2.0, b=0.05, c=0.3):
    return lambda x: a * math.exp(-b * x) + c


def simulate(loss, s_iter, e_iter, total, inter, t_train, t_p, t_c, t_infer):
    """Discrete-event simulation: inference j is issued at j*t_infer and served
    by the newest model that has ARRIVED by then (reading R11, arrival-inclusive).
    The model of checkpoint k (iteration s+k*inter <= e) arrives at
    k*(inter*t_train + t_p) + t_c; before the first arrival the initial model
    (iteration s) serves."""
    arrivals = []
    k = 1
    while s_iter + k * inter <= e_iter:
        arrivals.append((k * (inter * t_train + t_p) + t_c, loss(s_iter + k * inter)))
        k += 1
    total_loss, cur, a = 0.0, loss(s_iter), 0
    for j in range(total):
        t = j * t_infer
        while a < len(arrivals) and arrivals[a][0] <= t + 1e-12:
            cur = arrivals[a][1]
            a += 1
        total_loss += cur
    return total_loss


def alg2_cil_for(loss, s, e, total, i, tt, tp, tc, ti):
    """Alg. 2's t_l for one fixed interval i (lines 3-12), via S.cil."""
    t_l, rem = 0.0, total
    p_l = loss(s)
    c_iter, ver = s + i, 1
    while c_iter <= e:
        il, inf = S.cil(i, p_l, ver, rem, tt, tp, tc, ti)
        t_l, rem = t_l + il, rem - inf
        p_l = loss(c_iter)
        c_iter, ver = c_iter + i, ver + 1
    return t_l + p_l * rem


# ------------------------------------------------------------ worked examples
def test_fixed_interval_worked_example():
    g = GOLD
    L = _L(g["a"], g["b"], g["c"])
    bi, cil = S.fixed_interval(L, g["s_iter"], g["e_iter"], g["total_infers"], g["t_train"], g["t_p"], g["t_c"], g["t_infer"])
    assert bi == g["fixed"]["best_interval"]
    assert cil == pytest.approx(g["fixed"]["cil"], abs=1e-6)
    args = (g["s_iter"], g["e_iter"], g["total_infers"])
    t = (g["t_train"], g["t_p"], g["t_c"], g["t_infer"])
    assert alg2_cil_for(L, *args, 1, *t) == pytest.approx(g["fixed"]["cil_interval_1"], abs=1e-6)
    assert alg2_cil_for(L, *args, 40, *t) == pytest.approx(g["fixed"]["cil_interval_40"], abs=1e-6)


def test_greedy_worked_examples():
    g = GOLD
    L = _L(g["a"], g["b"], g["c"])
    t = (g["t_train"], g["t_p"], g["t_c"], g["t_infer"])
    sc, pc = S.greedy(L, g["s_iter"], g["e_iter"], g["total_infers"], 0.2, *t)
    assert sc == g["greedy_thresh_0.2"]["sched"]
    assert pc == pytest.approx(g["greedy_thresh_0.2"]["cil"], abs=1e-6)
    sc, _ = S.greedy(L, g["s_iter"], g["e_iter"], g["total_infers"], 0.05, *t)
    assert sc == g["greedy_thresh_0.05"]["sched"] and len(sc) == g["greedy_thresh_0.05"]["n"]


# -------------------------------------------------- Alg. 1+2 == simulation
@pytest.mark.parametrize("case", range(30))
def test_alg2_equals_discrete_event_simulation(case):
    rng = np.random.default_rng(case)
    ti = float(rng.choice([1.0, 0.5, 2.0]))
    tt = ti * int(rng.integers(1, 9))
    tp = ti * int(rng.integers(0, 6))
    tc = ti * int(rng.integers(0, 6))
    s = int(rng.integers(0, 5))
    e = s + int(rng.integers(1, 30))
    total = int(rng.integers(1, 800))
    L = _L(float(rng.uniform(0.5, 3)), float(rng.uniform(0.01, 0.3)), float(rng.uniform(0, 1)))
    for i in range(1, e - s + 1):
        a = alg2_cil_for(L, s, e, total, i, tt, tp, tc, ti)
        b = simulate(L, s, e, total, i, tt, tp, tc, ti)
        assert a == pytest.approx(b, rel=1e-12, abs=1e-9), (i, a, b)
    bi, ml = S.fixed_interval(L, s, e, total, tt, tp, tc, ti)
    sims = [simulate(L, s, e, total, i, tt, tp, tc, ti) for i in range(1, e - s + 1)]
    assert ml == pytest.approx(min(sims), rel=1e-12)
    assert bi == 1 + int(np.argmin(sims)) or sims[bi - 1] == pytest.approx(min(sims), rel=1e-12)


def test_greedy_schedule_cil_equals_simulation():
    """Alg. 3's predicted CIL == simulating its irregular schedule."""
    L = _L()
    tt, tp, tc, ti, total = 3.0, 2.0, 1.0, 1.0, 400
    sc, pc = S.greedy(L, 0, 60, total, 0.1, tt, tp, tc, ti)
    # arrivals of an irregular schedule: stall-inclusive training clock
    t, prev, arr = 0.0, 0, []
    for it in sc:
        t += (it - prev) * tt + tp
        arr.append((t + tc, L(it)))
        prev = it
    # Alg. 1 charges t_c only to the first interval (t_c overlaps later training),
    # i.e. arrival_k = sum of (interval*t_train + t_p) + t_c for every k.
    total_loss, cur, a = 0.0, L(0), 0
    for j in range(total):
        while a < len(arr) and arr[a][0] <= j * ti + 1e-12:
            cur = arr[a][1]
            a += 1
        total_loss += cur
    assert pc == pytest.approx(total_loss, rel=1e-12)


# --------------------------------------------------------------- Eq. 2 pins
@pytest.mark.parametrize("ckpt", [1, 2, 3, 7, 20])
def test_eq2_infers_sum_to_horizon(ckpt):
    tt, tp, tc, ti, tmax = 0.07, 0.03, 0.02, 0.005, 10.0
    tpr = ckpt * tt + tp
    cnm = math.floor((tmax - tc) / tpr)
    assert cnm >= 1
    tot = sum(S.infers_eq2(k, cnm, ckpt, tmax, tt, tp, tc, ti) for k in range(cnm + 1))
    assert tot == pytest.approx(tmax / ti, rel=1e-12)


def test_eq2_no_update_case():
    L = _L()
    # t_max too short for any model to arrive: cnm = 0 -> loss(0) * t_max / t_infer
    assert S.acc_loss(L, 5, 1.0, 1.0, 0.5, 0.2, 0.01) == pytest.approx(L(0) * 100.0)


def test_eq2_matches_alg2_when_training_outlasts_horizon():
    L = _L()
    tt, tp, tc, ti = 2.0, 1.0, 1.0, 1.0
    tmax = 300.0
    for ckpt in (1, 2, 5, 9):
        eq2 = S.acc_loss(lambda k: L(k), ckpt, tmax, tt, tp, tc, ti)
        alg = alg2_cil_for(L, 0, 10_000, int(tmax / ti), ckpt, tt, tp, tc, ti)
        assert eq2 == pytest.approx(alg, rel=1e-12)


def test_eq3_argmin():
    L = _L()
    best = S.ckpt_opt_eq3(L, 30, 500.0, 7.0, 3.0, 2.0, 1.0)
    vals = [S.acc_loss(L, c, 500.0, 7.0, 3.0, 2.0, 1.0) for c in range(1, 31)]
    assert best == 1 + int(np.argmin(vals))


# --------------------------------------------------------------- Eq. 1 pins
def test_eq1_get_iters():
    tt, tp = 1.0, 2.5
    for ckpt in (1, 3, 4):
        tpr = ckpt * tt + tp
        prev = -1
        for step in range(400):
            tk = step * 0.05
            x = S.get_iters(tk, ckpt, tt, tp)
            assert x >= prev  # reading R4 makes x' monotone in t_k
            prev = x
        for k in range(6):  # at each checkpoint boundary exactly k*ckpt iterations are done
            assert S.get_iters(k * tpr, ckpt, tt, tp) == k * ckpt
            # during the stall the iteration count does not move
            assert S.get_iters(k * tpr + ckpt * tt + 0.5 * tp, ckpt, tt, tp) == (k + 1) * ckpt


# --------------------------------------------------------- Alg. 2 special cases
def test_alg2_constant_loss_picks_smallest():
    bi, _ = S.fixed_interval(lambda x: 0.7, 0, 20, 300, 1.0, 1.0, 1.0, 1.0)
    assert bi == 1


def test_alg2_free_checkpoints_pick_every_iteration():
    bi, _ = S.fixed_interval(_L(), 0, 30, 1000, 1.0, 0.0, 0.0, 1.0)
    assert bi == 1


def test_alg2_expensive_checkpoints_pick_max_interval():
    bi, _ = S.fixed_interval(_L(), 0, 40, 100_000, 1.0, 100.0, 0.0, 1.0)
    assert bi == 40


def test_alg2_loop_bounds():
    """R2: intervals 1..(e-s) inclusive are all tried."""
    seen = []
    L = _L()
    S.fixed_interval(lambda x: (seen.append(x), L(x))[1], 3, 9, 50, 1.0, 0.0, 0.0, 1.0)
    assert max(seen) == 9 and 3 in seen


# ------------------------------------------------------------------ TLP pins
def test_tlp_recovers_noise_free_exp3():
    x = np.arange(60.0)
    y = 2.0 * np.exp(-0.05 * x) + 0.3
    fam, p, mses = S.fit_tlp(x, y)
    assert fam == S.EXP3
    assert p == pytest.approx([2.0, 0.05, 0.3], rel=1e-6)
    tl = GOLD["tlp_noise_free_exp3"]
    assert mses[S.EXP2] == pytest.approx(tl["mse_exp2"], rel=1e-2)
    assert mses[S.LIN2] == pytest.approx(tl["mse_lin2"], rel=1e-2)


def test_tlp_recovers_noise_free_exp2():
    x = np.arange(40.0)
    y = 1.7 * np.exp(-0.08 * x)
    fam, p, _ = S.fit_tlp(x, y)
    assert fam == S.EXP2
    assert p[:2] == pytest.approx([1.7, 0.08], rel=1e-6)


def test_tlp_lin2_equals_polyfit():
    rng = np.random.default_rng(5)
    x = np.arange(30.0)
    y = 3.0 - 0.04 * x + rng.normal(0, 0.01, 30)
    p, mse = S.fit_family(S.LIN2, x, y)
    ref = np.polyfit(x, y, 1)
    assert p[:2] == pytest.approx(ref, rel=1e-9)
    assert mse == pytest.approx(np.mean((np.polyval(ref, x) - y) ** 2), rel=1e-9)


def test_tlp_expd3_is_exp3_reparametrised():
    x = np.arange(50.0)
    y = 0.4 - (0.4 - 2.2) * np.exp(-0.07 * x)   # Expd3 with a=2.2, b=0.07, c=0.4
    fam, p, mses = S.fit_tlp(x, y)
    assert fam == S.EXP3  # ties go to the earlier family (reading R7)
    assert S.mse_equal(mses[S.EXP3], mses[S.EXPD3])
    pd, _ = S.fit_family(S.EXPD3, x, y)
    assert pd == pytest.approx([2.2, 0.07, 0.4], rel=1e-6)


def test_warmup_threshold_population_std():
    rng = np.random.default_rng(9)
    l = list(2.0 * np.exp(-0.05 * np.arange(40)) + rng.normal(0, 0.01, 40))
    d = [abs(b - a) for a, b in zip(l, l[1:])]
    assert S.warmup_threshold(l) == pytest.approx(statistics.fmean(d) + statistics.pstdev(d), rel=1e-12)


def test_schedule_pipeline_uses_bandwidths():
    x = np.arange(30.0)
    y = 2.0 * np.exp(-0.05 * x) + 0.3
    out = S.schedule(y, 0, 40, 500, 7.0, 1.0, s_model=3e9, bw_write=1e9, bw_read=1.5e9, algo=0)
    assert out["t_p"] == pytest.approx(3.0) and out["t_c"] == pytest.approx(2.0)
    assert out["family"] == S.EXP3 and out["best_interval"] == 4
    assert out["sched"] == list(range(4, 41, 4))
    g = S.schedule(y, 0, 40, 500, 7.0, 1.0, t_p=3.0, t_c=2.0, algo=1, thresh=0.2)
    assert g["sched"] == GOLD["greedy_thresh_0.2"]["sched"]
