"""NEXT-3 (P1157-1171, Fig. 14): client CPU cost and JCT of the completion wait,
measured in native code (paella_bench_wait): one thread submits ResNet-18 requests at a
fixed rate, a second thread waits with (a) a spinning poll, (b) PAELLA_HYBRID.  Prints
one JSON line per rate: the waiter's CPU utilisation and the client-observed JCT."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from paper_conf_sosp_ngd023_b200 import _lib as L  # noqa: E402
from workload import archs, rng  # noqa: E402

rates = [float(r) for r in (sys.argv[1:] or ["1000", "4000"])]
g = archs.build("resnet18")
e = L.Engine(num_clients=1, lookahead=3, slack=1184, launch_threads=4)
mid = e.register_model(g, rng.model_params(g))
info = e.model_info(mid)
stride = (info["input_bytes"] + info["output_bytes"] + 4095) // 4096 * 4096
_, reg = e.region(0)
x = rng.image(g, 0)
for s in range(64):
    reg[s * stride:s * stride + x.nbytes] = np.frombuffer(x.tobytes(), np.uint8)
for rate in rates:
    n = int(min(20000, rate * 3))
    row = {"model": "resnet18", "req_s": rate, "requests": n}
    for label, flags in (("spin", 0), ("hybrid", L.HYBRID)):
        j, cpu = e.bench_wait(0, mid, n, 1e9 / rate, flags, stride, 64)
        j = j[j > 0] / 1e3
        row[label] = {"waiter_cpu_util": round(cpu, 3), "jct_mean_us": round(float(j.mean()), 1),
                      "jct_p50_us": round(float(np.percentile(j, 50)), 1),
                      "jct_p99_us": round(float(np.percentile(j, 99)), 1)}
    print(json.dumps(row), flush=True)
e.shutdown()
