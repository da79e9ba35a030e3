"""bench.py contract checks that need no GPU: the module imports, every stage
it calls exists, and the reference arm prints the required keys."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def test_bench_functions_exist():
    import bench
    for fn in ("run_update_bench", "run_e2e", "c3_concurrent", "c5_schedule", "event_floor_us", "cpu_baseline",
               "xproc_arm", "xproc_e2e", "ce_baseline", "gpu_arm", "reference_arm", "main", "ncu_traffic",
               "load_peaks"):
        assert callable(getattr(bench, fn)), fn


def test_reference_arm_json_line():
    r = subprocess.run([sys.executable, "bench.py", "--impl", "reference", "--steps", "3", "--warmup", "3",
                        "--cpu-budget", "0.5"], cwd=ROOT, stdout=subprocess.PIPE, stderr=subprocess.PIPE,
                       text=True, timeout=300)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.strip()]
    assert len(lines) == 1
    d = json.loads(lines[0])
    for k in ("impl", "metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "cpu_baseline", "e2e", "config"):
        assert k in d, k
    assert d["impl"] == "reference" and d["higher_is_better"] is False and d["value"] > 0
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["cpu_baseline"]["kind"] == "oracle"


def _json_lines(out):
    return [json.loads(l) for l in out.splitlines() if l.strip().startswith("{")]


def test_gpus_n_self_launches_ranks():
    """`bench.py --gpus 2` without a launcher starts 2 ranks
    itself (torch.distributed.run on 127.0.0.1); on this CPU box the ranks
    rendezvous over gloo, reduce over ranks and rank 0 prints ONE line with
    n_gpus = 2 and no number (there is no GPU to measure)."""
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    r = subprocess.run([sys.executable, "bench.py", "--gpus", "2", "--oversubscribe", "--steps", "3", "--warmup", "3"],
                       cwd=ROOT, stdout=subprocess.PIPE, stderr=subprocess.PIPE, text=True, timeout=300, env=env)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = _json_lines(r.stdout)
    assert len(lines) == 1, r.stdout[-2000:]
    d = lines[0]
    assert d["n_gpus"] == 2 and d["ranks_seen"] == 2 and d["value"] is None and "unavailable" in d


def test_gpus_n_fails_loudly_without_gpus():
    """--gpus 2 with fewer visible GPUs and no --oversubscribe: non-zero exit,
    no JSON line (never a silent 1-GPU measurement)."""
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    r = subprocess.run([sys.executable, "bench.py", "--gpus", "2", "--steps", "3"], cwd=ROOT, stdout=subprocess.PIPE,
                       stderr=subprocess.PIPE, text=True, timeout=120, env=env)
    assert r.returncode != 0 and not _json_lines(r.stdout)
    assert "--oversubscribe" in r.stderr


def test_gpus_must_match_world_size():
    env = dict(os.environ, WORLD_SIZE="1", RANK="0", LOCAL_RANK="0")
    r = subprocess.run([sys.executable, "bench.py", "--gpus", "2", "--steps", "3"], cwd=ROOT, stdout=subprocess.PIPE,
                       stderr=subprocess.PIPE, text=True, timeout=120, env=env)
    assert r.returncode != 0 and "WORLD_SIZE=1" in r.stderr


def test_reference_arm_under_two_ranks():
    """--impl reference at N = 2: rank 0 alone runs the oracle with the N = 2
    config (1 -> 1); the other rank exits without work; one line."""
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    r = subprocess.run([sys.executable, "bench.py", "--impl", "reference", "--gpus", "2", "--oversubscribe",
                        "--steps", "3", "--warmup", "3", "--cpu-budget", "0.5"], cwd=ROOT, stdout=subprocess.PIPE,
                       stderr=subprocess.PIPE, text=True, timeout=300, env=env)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = _json_lines(r.stdout)
    assert len(lines) == 1 and lines[0]["impl"] == "reference" and lines[0]["n_gpus"] == 2


def test_cpu_baseline_p_threads():
    """the oracle on 1 thread and on P threads (disjoint tensor
    subsets), with the core count stated."""
    import bench
    import synth
    cb = bench.cpu_baseline(synth, "ptychonn", budget_s=0.3, max_updates=5)
    assert cb["cores"] == 1 and cb["kind"] == "oracle" and cb["value"] > 0
    p = cb["p_threads"]
    assert p["cores"] >= 1 and p["value"] > 0 and p["cores"] <= cb["cpu"]["affinity_cores"]


def test_summarize_fanout_math_and_parity():
    """The N > 1 line's per-fan-out summary: value = max over ranks of the
    device windows, f_NVL = S / L / 900 GB/s, parity requires every consumer's
    golden-seal match, byte match and final version; an unsupported fan-out
    (NVLS without multicast) is reported as such."""
    import bench
    S = 102228128
    ver_ok = {"seals_ok": True, "bytes_ok": True, "chunks": 49, "version": 9, "version_ok": True}
    prod = {"lat": [0.2, 0.2, 0.2], "host": [0.21] * 3, "inst": [], "verify": dict(ver_ok, bytes_ok=None),
            "s_packed": S}
    cons = {"lat": [], "host": [], "inst": [150.0, 160.0, 170.0], "verify": ver_ok, "s_packed": S}
    r = bench.summarize_fanout([prod, cons], S)
    assert abs(r["latency_ms"] - 0.2) < 1e-12
    assert abs(r["nvlink_frac"] - S / 0.2e-3 / 1e9 / 900.0) < 1e-4
    assert r["install_kernel_us_per_consumer"] == [160.0] and r["parity_ok"] is True
    slow = dict(cons, inst=[300.0] * 3)  # a consumer whose install window exceeds the producer's
    assert abs(bench.summarize_fanout([prod, slow], S)["latency_ms"] - 0.3) < 1e-12
    bad = dict(cons, verify=dict(ver_ok, seals_ok=False))
    assert bench.summarize_fanout([prod, bad], S)["parity_ok"] is False
    un = bench.summarize_fanout([{"unsupported": "VIPER_E_UNSUPPORTED: no multicast"}] * 2, S)
    assert "unsupported" in un


def test_xproc_line_survives_a_failed_headline():
    """The N > 1 line prints even when the headline fan-out failed (it once
    raised KeyError and lost the line): value null, no roofline, the error
    kept under `fanouts`; with a verified headline, value = its latency and
    the NVLink fraction follows from it."""
    import types

    import bench
    S = 102228128
    args = types.SimpleNamespace(steps=3, warmup=3)
    conc = [{"publishes": 10}, {"torn": 0, "regress": 0, "views_idle": 100.0, "views_busy": 90.0, "installs": 10}]
    e2e = {"h2d": S, "d2h": 784}
    t = [0.5, 0.4, 2.0, 0.0]
    clocks = {"sm_mhz": 1965.0, "sm_max_mhz": 1965.0, "reasons": []}
    failed = bench.summarize_fanout([{"lat": [], "host": [], "inst": [], "errors": ["publish(1): VIPER_E_TIMEOUT"],
                                      "verify": {}, "s_packed": S}, {"lat": [], "host": [], "inst": [], "errors": [],
                                                                     "verify": {}, "s_packed": S}], S)
    line = bench.xproc_line(args, 2, "resnet50", S, 2, False, "direct", {"direct": failed}, conc, t, e2e, clocks)
    json.dumps(line)
    assert line["value"] is None and line["roofline"] is None and line["parity_ok"] is False
    assert line["fanouts"]["direct"]["error"] and line["n_gpus"] == 2
    ver_ok = {"seals_ok": True, "bytes_ok": True, "chunks": 49, "version": 7, "version_ok": True}
    good = bench.summarize_fanout([{"lat": [0.15] * 3, "host": [0.16] * 3, "inst": [], "s_packed": S,
                                    "verify": dict(ver_ok, bytes_ok=None)},
                                   {"lat": [], "host": [], "inst": [120.0] * 3, "verify": ver_ok, "s_packed": S}], S)
    line = bench.xproc_line(args, 2, "resnet50", S, 2, False, "direct", {"direct": good, "dram": failed}, conc, t,
                            e2e, clocks)
    json.dumps(line)
    assert abs(line["value"] - 0.15) < 1e-12 and line["parity_ok"] is True
    assert abs(line["roofline"]["frac"] - S / 0.15e-3 / 1e9 / 900.0) < 1e-3
    assert line["dram_over_gpu"] is None and line["concurrent_acquire"]["torn_views"] == 0


def test_bench_fanout_codes_match_the_abi():
    """bench.py's fan-out names map to include/viper.h's VIPER_FANOUT_* codes
    (through the binding's constants), and the baselines never headline."""
    import bench
    from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V
    assert bench.FANOUTS["direct"] == V.FANOUT_DIRECT and bench.FANOUTS["chain"] == V.FANOUT_CHAIN
    assert bench.FANOUTS["sa"] == V.FANOUT_SCATTER_ALLGATHER and bench.FANOUTS["nvls"] == V.FANOUT_NVLS
    assert bench.FANOUTS["push"] == V.FANOUT_PUSH and bench.FANOUTS["nccl"] == V.FANOUT_NCCL
    assert bench.FANOUTS["ce"] == V.FANOUT_CE and bench.FANOUTS["dram"] < 0
    hdr = open(os.path.join(ROOT, "include", "viper.h")).read()
    for name, code in (("NVLS", 3), ("PUSH", 4), ("NCCL", 100), ("CE", 101)):
        assert f"VIPER_FANOUT_{name} = {code}" in hdr
