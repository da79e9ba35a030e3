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
