"""Diagnosis: the C-3 mix's device-only saturation rate (X_dev: CUDA graphs of the mix on
32 streams, no dispatcher) next to its isolated latency (summed instrumented kernel
times) and device work (summed CTAs), for the current environment's planner/autotuner
switches (PAELLA_M64, PAELLA_NO_TMA_B, PAELLA_SPLIT_GAIN, ...).  One JSON line.  No oracle."""
import json
import os
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from paper_conf_sosp_ngd023_b200 import _lib as L  # noqa: E402
from workload import archs, rng  # noqa: E402

names = ["resnet50", "densenet121", "inception_v3", "mobilenet_v2"]
res = {"env": {k: v for k, v in os.environ.items() if k.startswith("PAELLA_")}}
with L.Engine(num_clients=1) as e:
    mids = []
    for name in names:
        g = archs.build(name)
        mid = e.register_model(g, rng.model_params(g), name=name)
        mids.append(mid)
        ks = e.kernels(mid)
        ti = e.time_kernels(mid, instrumented=True, reps=50)
        res[name] = {"instr_us": round(float(ti.sum()) / 1e3, 1),
                     "ctas": int(sum(int(np.prod(k["grid"])) if isinstance(k["grid"], (list, tuple)) else int(k["grid"])
                                     for k in ks))}
    seq = np.random.default_rng(7).integers(0, len(names), 2000)
    res["x_dev"] = [round(e.bench_xdev(mids, seq, streams=32), 1) for _ in range(3)]
print(json.dumps(res), flush=True)
