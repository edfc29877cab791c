"""ORACLE script: writes workload/data/lsuv_scales.json (the stored LSUV factors).

Calls only ``oracle/`` (and the neutral ``workload`` generators).  Recipe: SURVEY.md
§8(c) C1 step 3.  Run:  python -m oracle.make_lsuv_scales
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

from workload import archs, rng  # noqa: E402
from oracle.infer import lsuv_scales  # noqa: E402


def main():
    out = {}
    for name in archs.MODELS:
        g = archs.build(name)
        out[name] = lsuv_scales(g, rng.raw_params(g), rng.calibration_input(g))
        print(name, len(out[name]), file=sys.stderr)
    os.makedirs(os.path.dirname(rng.SCALES_PATH), exist_ok=True)
    with open(rng.SCALES_PATH, "w") as f:
        json.dump(out, f, indent=0, sort_keys=True)


if __name__ == "__main__":
    main()
