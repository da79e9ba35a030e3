"""Summarise ncu reports (raw page) and launch lists into profiles/ (run here, no GPU)."""
import csv
import io
import json
import subprocess
import sys

METRICS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
           "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
           "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread", "launch__grid_size",
           "launch__block_size", "lts__t_sectors_srcunit_tex_op_read_lookup_hit.sum",
           "lts__t_sectors_srcunit_tex_op_read_lookup_miss.sum",
           "smsp__pcsamp_warps_issue_stalled_long_scoreboard", "smsp__pcsamp_warps_issue_stalled_membar",
           "smsp__pcsamp_sample_count"]
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "us": 1e-6, "ms": 1e-3, "ns": 1e-9, "s": 1}


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], stdout=subprocess.PIPE, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {"kernel": r[hdr.index("Kernel Name")]}
        for m in METRICS:
            if m in hdr:
                i = hdr.index(m)
                try:
                    v = float(r[i].replace(",", ""))
                except ValueError:
                    continue
                u = units[i]
                d[m] = v * SCALE[u] if u in SCALE else v
                d[m + ".unit"] = "B" if u in ("byte", "Kbyte", "Mbyte", "Gbyte") else ("s" if u in ("us", "ms", "ns", "s") else u)
        res.append(d)
    return res


def launches(path):
    rows = list(csv.reader(open(path)))
    start = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    hdr = rows[start]
    out = {}
    for r in rows[start + 1:]:
        if len(r) < len(hdr):
            continue
        d = dict(zip(hdr, r))
        if d.get("Metric Name") != "gpu__time_duration.sum":
            continue
        name = d["Kernel Name"]
        k = name.split("(")[0].replace("void ", "").split("::")[-1] if "(" in name else name
        v = float(d["Metric Value"].replace(",", ""))
        scale = {"ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3}.get(
            d.get("Metric Unit", "us"), 1.0)
        out.setdefault(k, []).append(v * scale)
    return {k: {"launches": len(v), "total_us": round(sum(v), 3), "mean_us": round(sum(v) / len(v), 3)}
            for k, v in out.items()}


if __name__ == "__main__":
    mode, *args = sys.argv[1:]
    if mode == "raw":
        print(json.dumps({a: raw(a) for a in args}, indent=1))
    else:
        print(json.dumps(launches(args[0]), indent=1))
