"""Write profiles/ncu_traffic.json (per-launch DRAM traffic of each kernel from
the committed `ncu --set full` summaries) -- read by bench.py's roofline
`traffic` field.  Usage: python tools/ncu_traffic.py profiles/r01/ncu_full_summary_s2.json"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def main(summary):
    d = json.load(open(summary))
    path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    out = json.load(open(path)) if os.path.exists(path) else {}  # merge: newer captures replace their rows
    for rep, kernels in d.items():
        cfg = rep.replace(".ncu-rep", "").split("_")[-1]  # ..._<cfg>
        cfg = {"r50": "resnet50", "vit": "vit_b16", "gpt2": "gpt2_xl"}.get(cfg, cfg)
        for k in kernels:
            name = k["kernel"].split("::")[-1].split("(")[0]
            rd, wr = k["dram__bytes_read.sum"], k["dram__bytes_write.sum"]
            out[f"{name}:{cfg}"] = {"dram_read_bytes": rd, "dram_write_bytes": wr, "traffic_bytes": rd + wr,
                                    "gpu_time_us_cold": round(k["gpu__time_duration.sum"] * 1e6, 3),
                                    "grid": k.get("launch__grid_size"), "block": k.get("launch__block_size"),
                                    "registers": k.get("launch__registers_per_thread"),
                                    "source": f"{os.path.relpath(summary, ROOT)} ({rep})"}
    with open(path, "w") as f:
        json.dump(out, f, indent=1)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main(sys.argv[1])
