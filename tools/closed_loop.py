"""N2 closed loop: viper_schedule driven by the engine's measured
costs, a synthetic trainer publishing at the scheduled iterations, a serving
thread acquiring the latest model, CIL accounted on the measured timeline.

    python tools/closed_loop.py [--out profiles/r01/closed_loop.json] [--quick]
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icpp_yecrbypnmskn24_b200 import closed_loop as CL  # noqa: E402
from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V  # noqa: E402

CASES = [
    # the GPU tier on GPT-2 XL (3.1 GB): t_p ~ pack, comparable to a 2 ms iteration
    dict(model="gpt2_xl", tier=V.TIER_GPU, mode=V.ASYNC, t_train=2e-3, t_infer=5e-4, s_iter=50, e_iter=800),
    dict(model="gpt2_xl", tier=V.TIER_GPU, mode=V.SYNC, t_train=2e-3, t_infer=5e-4, s_iter=50, e_iter=800),
    # the pinned-DRAM tier on the same model: t_p, t_c ~ 10x an iteration
    dict(model="gpt2_xl", tier=V.TIER_DRAM, mode=V.ASYNC, t_train=1e-2, t_infer=2e-3, s_iter=50, e_iter=400),
]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default="profiles/r01/closed_loop.json")
    ap.add_argument("--quick", action="store_true")
    a = ap.parse_args()
    res = []
    cases = CASES[:1] if a.quick else CASES
    for c in cases:
        r = CL.run(**c)
        res.append(r)
        print(json.dumps(r), flush=True)
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    with open(a.out, "w") as f:
        json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
