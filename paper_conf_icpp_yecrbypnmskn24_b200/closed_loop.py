"""N2: the IPP schedule driving the engine, closed loop.

The paper's IPP (s4.3) picks checkpoint iterations from a fitted
training-loss curve and the two transfer costs t_p (producer stall,
P:1346-1352) and t_c (consumer load).  This module runs that
loop end to end on one GPU:

1. A synthetic trainer.  One iteration is a GPU busy kernel of about
   `t_train` plus a VGEN write of one marker tensor, ended by a stream
   synchronize (the loss read-back).  The loss it "observes" at iteration x is
   a seeded Exp3 curve L(x) = a e^{-bx} + c, with Gaussian
   noise on the warm-up observations.
2. Calibration.  t_train, t_p and t_c are measured on the engine:
   * t_p = (iteration with a publish) - (iteration without);
   * t_c = the consumer's install callback - the end of the publishing iteration.
3. viper_schedule.  It gets the s_iter warm-up losses and the measured
   costs, and runs Alg. 2 (fixed interval) and Alg. 3 (greedy).
4. The rest of training.  Iterations s_iter..e_iter run, and the model is
   published (version = iteration) at each scheduled iteration.  A serving
   thread issues inference j at t0 + j*t_infer, for
   total_infers = (e_iter - s_iter) t_train / t_infer inferences.  Each one
   acquires the latest installed version and releases it.

CIL (cumulative inference loss, Eq. 2) is accounted three ways:
* `predicted`: the schedule's own model.  It uses the fitted curve on the
  ideal timeline (arrival of checkpoint k = sum of (interval t_train + t_p)
  + t_c, Alg. 1).
* `timeline`: the s8(c) simulation on the MEASURED install times, with the
  true curve (R11: arrival-inclusive).
* `served`: the sum of L(version) over what the serving thread actually
  acquired.

Baseline policies run beside the IPP: publish every iteration, fixed
intervals, and never (only the initial model serves).

Host-side orchestration only.  Every byte still moves through libviper's
kernels (V.Model.publish / acquire_latest / release).
"""
from __future__ import annotations

import math
import threading
import time

import numpy as np


def cil_from_arrivals(l0: float, arrivals, total_infers: int, t_infer: float) -> float:
    """Inference j (issued at j*t_infer) is served by the newest model that
    arrived at or before that time (reading R11, arrival-inclusive).  Before
    the first arrival, the initial model with loss l0 serves.
    arrivals: iterable of (t_arrival, loss), in publish order."""
    arr = sorted(arrivals, key=lambda a: a[0])
    total, cur, a = 0.0, float(l0), 0
    for j in range(int(total_infers)):
        t = j * t_infer
        while a < len(arr) and arr[a][0] <= t + 1e-12:
            cur = float(arr[a][1])
            a += 1
        total += cur
    return total


def ideal_arrivals(sched, s_iter: int, t_train: float, t_p: float, t_c: float, loss):
    """Alg. 1's timeline for an arbitrary schedule (list of iterations):
    training pays t_p per checkpoint, and a model lands t_c after its stall ends."""
    t, prev, out = 0.0, s_iter, []
    for it in sched:
        t += (it - prev) * t_train + t_p
        out.append((t + t_c, loss(it)))
        prev = it
    return out


class LossCurve:
    """Seeded Exp3 training-loss curve, L(x) = a e^{-bx} + c."""

    def __init__(self, a=2.0, b=0.005, c=0.5, noise=0.01, seed=5):
        self.a, self.b, self.c, self.noise = a, b, c, noise
        self.rng = np.random.default_rng(seed)

    def __call__(self, x):
        return self.a * math.exp(-self.b * x) + self.c

    def observe(self, x):
        return self(x) + (self.rng.normal(0.0, self.noise) if self.noise > 0 else 0.0)


class SyntheticTrainer:
    """One iteration = busy kernel (~t_train) + VGEN write of the marker
    tensor (its bytes name the iteration) + stream synchronize."""

    def __init__(self, tensors, specs, seed, t_train, marker=0):
        import torch
        from synth import gpu as G
        self.torch, self.G = torch, G
        self.tensors, self.specs, self.seed, self.marker = tensors, specs, seed, marker
        self.stream = torch.cuda.current_stream()
        self.cycles = self._cycles_for(t_train)

    def _cycles_for(self, seconds):
        torch = self.torch
        probe = 20_000_000
        torch.cuda._sleep(probe // 10)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        torch.cuda._sleep(probe)
        e1.record()
        e1.synchronize()
        hz = probe / (e0.elapsed_time(e1) * 1e-3)
        return max(int(seconds * hz), 1)

    def work(self, it: int):
        self.torch.cuda._sleep(self.cycles)
        m = self.marker
        self.G.fill(self.tensors[m], self.seed, it, m, self.specs[m][1])

    def step(self, it: int, publish=None):
        """Run iteration `it`; `publish(it)` (if given) right after its work,
        before the read-back.  Returns the host time at the iteration's end."""
        self.work(it)
        if publish is not None:
            publish(it)
        self.stream.synchronize()
        return time.perf_counter()


class _Arrivals:
    def __init__(self):
        self.t = {}
        self.lock = threading.Lock()

    def __call__(self, version, status):
        if status == 0:
            now = time.perf_counter()
            with self.lock:
                self.t.setdefault(version, now)

    def wait(self, version, timeout=30.0):
        """The callback runs after the swap that wait_installed observes."""
        end = time.perf_counter() + timeout
        while version not in self.t:
            if time.perf_counter() > end:
                raise TimeoutError(f"no install callback for version {version}")
            time.sleep(1e-5)
        return self.t[version]


def _serve(cons, t0, total, t_infer, out_v, out_late):
    for j in range(total):
        target = t0 + j * t_infer
        d = target - time.perf_counter()
        if d > 2e-4:
            time.sleep(d - 1e-4)
        while time.perf_counter() < target:
            pass
        view = cons.acquire_latest()
        out_late[j] = time.perf_counter() - target
        out_v[j] = view.version
        cons.release(view)


class ClosedLoop:
    """Producer + consumer of one synthetic workload in this process."""

    def __init__(self, model="gpt2_xl", tier=0, mode=1, t_train=2e-3, t_infer=5e-4, s_iter=50, e_iter=800,
                 curve=None):
        import synth
        from synth import gpu as G
        from . import viper as V
        self.V, self.G = V, G
        self.specs = synth.model_specs(model)
        self.seed = synth.SEEDS[model]
        self.model, self.tier, self.mode = model, tier, mode
        self.t_train_target, self.t_infer = t_train, t_infer
        self.s_iter, self.e_iter = s_iter, e_iter
        self.curve = curve or LossCurve()
        self.pt, self.ct = G.alloc_model(self.specs), G.alloc_model(self.specs)
        G.fill_model(self.pt, self.specs, self.seed, 1)
        self.arr = _Arrivals()
        self.prod = V.Model(model + "_loop", V.PRODUCER, self.pt, tier=tier, mode=mode)
        self.cons = V.Model(model + "_loop", V.CONSUMER, self.ct, tier=tier)
        self.cons.subscribe(self.arr)
        self.trainer = SyntheticTrainer(self.pt, self.specs, self.seed, t_train)
        self.base = 0          # versions of one policy run: base + iteration
        self.total_infers = int(round((e_iter - s_iter) * t_train / t_infer))

    # ---------------------------------------------------------- calibration
    def _pub(self, it):
        self.prod.publish(self.base + it, stream=self.trainer.stream)

    def _next_base(self):
        self.base += 1_000_000
        return self.base

    def calibrate(self, reps=12):
        """Measured t_train, t_p, t_c (medians) on this engine and workload."""
        tr = self.trainer
        self._next_base()
        for it in range(3):
            tr.step(it, self._pub)
        self.cons.wait_installed(self.base + 2)
        plain, pub, lag = [], [], []
        for r in range(reps):
            t0 = time.perf_counter()
            tr.step(10 + 2 * r)
            t1 = time.perf_counter()
            te = tr.step(11 + 2 * r, self._pub)
            self.cons.wait_installed(self.base + 11 + 2 * r)
            plain.append(t1 - t0)
            pub.append(te - t1)
            lag.append(max(self.arr.wait(self.base + 11 + 2 * r) - te, 0.0))
        # back-to-back publishes: the tier's steady-state stall.  With the DRAM
        # tier a publish waits for the previous snapshot's D2H to drain
        # (reading R22), which an isolated publish never sees.
        steady, t_prev = [], time.perf_counter()
        for r in range(reps):
            te = tr.step(100 + r, self._pub)
            steady.append(te - t_prev)
            t_prev = te
        self.cons.wait_installed(self.base + 100 + reps - 1)
        t_train = float(np.median(plain))
        t_p_iso = max(float(np.median(pub)) - t_train, 0.0)
        t_p_steady = max(float(np.median(steady[2:])) - t_train, 0.0)
        self.costs = {"t_train": t_train, "t_p": max(t_p_iso, t_p_steady), "t_c": float(np.median(lag)),
                      "t_p_isolated": t_p_iso, "t_p_back_to_back": t_p_steady}
        return self.costs

    # ------------------------------------------------------------- schedule
    def plan(self, thresh=-1.0):
        c = self.costs
        xs = list(range(self.s_iter))
        self.warm = [self.curve.observe(x) for x in xs]
        kw = dict(s_iter=self.s_iter, e_iter=self.e_iter, total_infers=self.total_infers, t_train=c["t_train"],
                  t_infer=self.t_infer, t_p=c["t_p"], t_c=c["t_c"], x=[float(x) for x in xs])
        self.fixed = self.V.schedule(self.warm, algo=self.V.SCHED_FIXED, **kw)
        self.greedy = self.V.schedule(self.warm, algo=self.V.SCHED_GREEDY, thresh=thresh, **kw)
        return self.fixed, self.greedy

    def predicted_loss(self, x):
        f, p = self.fixed["family"], self.fixed["params"]
        a, b, c = p
        return [a * math.exp(-b * x), a * math.exp(-b * x) + c, a * x + b, c - (c - a) * math.exp(-b * x)][f]

    # ------------------------------------------------------------------ run
    def run_policy(self, sched):
        """Train s_iter+1..e_iter, publishing at the iterations in `sched`,
        while the serving thread issues total_infers inferences."""
        base = self._next_base()
        s, e, tr = self.s_iter, self.e_iter, self.trainer
        tr.step(s, self._pub)                      # the initial model (iteration s) serves first
        self.cons.wait_installed(base + s)
        want = set(sched)
        total = self.total_infers
        served = np.zeros(total, dtype=np.int64)
        late = np.zeros(total, dtype=np.float64)
        t0 = time.perf_counter() + 2e-3
        th = threading.Thread(target=_serve, args=(self.cons, t0, total, self.t_infer, served, late))
        th.start()
        while time.perf_counter() < t0:
            pass
        ends = {}
        for it in range(s + 1, e + 1):
            ends[it] = tr.step(it, self._pub if it in want else None) - t0
        t_train_end = time.perf_counter() - t0
        th.join()
        if want:
            self.cons.wait_installed(base + max(want), timeout_us=30_000_000)
            self.arr.wait(base + max(want))
        L = self.curve
        arrivals = [(self.arr.t[base + it] - t0, L(it)) for it in sorted(want) if base + it in self.arr.t]
        sv = served - base
        versions_ok = bool(np.all(np.diff(sv) >= 0)) and set(sv.tolist()) <= (want | {s})
        c = self.costs
        return {
            "n_publish": len(want),
            "n_installed": len(arrivals),
            "train_s": round(t_train_end, 4),
            "predicted_cil": cil_from_arrivals(self.predicted_loss(s), ideal_arrivals(
                sorted(want), s, c["t_train"], c["t_p"], c["t_c"], self.predicted_loss), total, self.t_infer),
            "model_cil": cil_from_arrivals(L(s), ideal_arrivals(sorted(want), s, c["t_train"], c["t_p"], c["t_c"], L),
                                           total, self.t_infer),
            "timeline_cil": cil_from_arrivals(L(s), arrivals, total, self.t_infer),
            "served_cil": float(sum(L(int(v)) for v in sv)),
            "served_versions": int(len(set(sv.tolist()))),
            "versions_monotone_and_published": versions_ok,
            "serve_lateness_us_p50": round(float(np.median(late)) * 1e6, 1),
            "serve_lateness_us_p99": round(float(np.percentile(late, 99)) * 1e6, 1),
        }

    def best_interval_true_curve(self):
        """The interval Alg. 2 would pick if it knew the TRUE curve (same
        measured costs), for judging the fitted schedule."""
        c, s, e, L = self.costs, self.s_iter, self.e_iter, self.curve
        best, best_v = None, math.inf
        for i in range(1, e - s + 1):
            v = cil_from_arrivals(L(s), ideal_arrivals(list(range(s + i, e + 1, i)), s, c["t_train"], c["t_p"],
                                                       c["t_c"], L), self.total_infers, self.t_infer)
            if v < best_v:
                best, best_v = i, v
        return best, best_v

    def close(self):
        self.cons.close()
        self.prod.close()


def run(model="gpt2_xl", tier=0, mode=1, t_train=2e-3, t_infer=5e-4, s_iter=50, e_iter=800, fixed=(1, 10, 100),
        curve=None, greedy=True, true_best=True):
    """Calibrate, schedule, run the IPP policies and the baselines.  Returns a dict."""
    loop = ClosedLoop(model, tier, mode, t_train, t_infer, s_iter, e_iter, curve)
    try:
        costs = loop.calibrate()
        fx, gr = loop.plan()
        out = {"model": model, "tier": ["gpu", "dram"][tier], "mode": ["sync", "async"][mode],
               "s_iter": s_iter, "e_iter": e_iter, "t_infer_s": t_infer, "total_infers": loop.total_infers,
               "measured": {k: round(v, 7) for k, v in costs.items()},
               "schedule": {"family": ["Exp2", "Exp3", "Lin2", "Expd3"][fx["family"]],
                            "params": [round(p, 6) for p in fx["params"]], "best_interval": fx["best_interval"],
                            "alg2_predicted_cil": fx["predicted_cil"], "greedy_checkpoints": len(gr["sched"]),
                            "alg3_predicted_cil": gr["predicted_cil"]},
               "policies": {}}
        pol = {f"ipp_fixed_{fx['best_interval']}": list(range(s_iter + fx["best_interval"], e_iter + 1,
                                                               fx["best_interval"]))}
        if greedy:
            pol["ipp_greedy"] = list(gr["sched"])
        for i in fixed:
            pol.setdefault(f"fixed_{i}", list(range(s_iter + i, e_iter + 1, i)))
        pol["never"] = []
        for name, sc in pol.items():
            out["policies"][name] = loop.run_policy(sc)
        if true_best:
            bi, bv = loop.best_interval_true_curve()
            out["true_curve_best_interval"] = bi
            out["true_curve_best_model_cil"] = bv
        return out
    finally:
        loop.close()
