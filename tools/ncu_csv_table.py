"""Median per-kernel duration and DRAM bytes from `ncu --metrics ... --csv`
logs (one file per run), with the fraction of the measured HBM peak at 2S.
Usage: python tools/ncu_csv_table.py 'gpurun_out/idsweep_*.csv'"""
import csv
import glob
import io
import json
import os
import re
import statistics
import sys

S = {"ptychonn": 4616840, "resnet50": 102228128, "vit_b16": 173135312, "gpt2_xl": 3115222400,
     "llama3_8b": 16060522496}
T_SCALE = {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3}
B_SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}


def parse(path):
    txt = open(path).read()
    i = txt.find('"ID"')
    if i < 0:
        return None
    rows = list(csv.reader(io.StringIO(txt[i:])))
    hdr = rows[0]
    d = {}
    for r in rows[1:]:
        if len(r) < len(hdr):
            continue
        x = dict(zip(hdr, r))
        k = x["Kernel Name"].split("(")[0].split("::")[-1]
        v = float(x["Metric Value"].replace(",", ""))
        u = x["Metric Unit"]
        v *= T_SCALE.get(u, B_SCALE.get(u, 1.0))
        d.setdefault(k, {}).setdefault(x["Metric Name"], []).append(v)
    return d


def main(pattern, peak=None):
    if peak is None:
        try:
            peak = json.load(open(os.path.join(os.path.dirname(__file__), "..", "MEASURED_PEAKS.json")))["hbm_gbs"]
        except Exception:
            peak = 6470.2
    out = []
    for f in sorted(glob.glob(pattern)):
        d = parse(f)
        cfg = next((c for c in S if f"_{c}_" in os.path.basename(f)), None)
        if not d or not cfg:
            print(f"{f}: no data")
            continue
        for k, m in d.items():
            t = statistics.median(m["gpu__time_duration.sum"])
            rd = statistics.median(m.get("dram__bytes_read.sum", [0]))
            wr = statistics.median(m.get("dram__bytes_write.sum", [0]))
            frac = 2 * S[cfg] / (t * 1e-6) / 1e9 / peak
            row = {"file": os.path.basename(f), "kernel": k, "config": cfg, "us": round(t, 2),
                   "frac_2S": round(frac, 4), "dram_read_MB": round(rd / 1e6, 1), "dram_write_MB": round(wr / 1e6, 1)}
            out.append(row)
            print(f"{row['file']:52s} {k:28s} {t:9.2f} us  2S-frac {frac:.3f}  rd {rd/1e6:8.1f} MB  wr {wr/1e6:8.1f} MB")
    return out


if __name__ == "__main__":
    main(sys.argv[1])
