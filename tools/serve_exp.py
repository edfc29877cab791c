"""Experiment: unloaded JCT and saturation of serving variants (no oracle)."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
from paper_conf_sosp_ngd023_b200 import _lib as L
from workload import archs, rng, traces

names = ["resnet18", "mobilenet_v2", "squeezenet1_1"]
specs = [(archs.build(n), None) for n in names]
specs = [(g, rng.model_params(g)) for g, _ in specs]
pool = [[rng.image(g, i) for i in range(8)] for g, _ in specs]
slots, stride = 128, 1 << 20
variants = json.loads(sys.argv[1]) if len(sys.argv) > 1 else [
    {"naive": True, "instrument": False, "launch_threads": 2},
    {"lookahead": 0, "launch_threads": 2},
    {"lookahead": 1, "launch_threads": 2},
    {"lookahead": 2, "launch_threads": 2},
    {"lookahead": 1, "launch_threads": 0},
    {"lookahead": 1, "launch_threads": 4},
    {"lookahead": 2, "launch_threads": 4},
]
for v in variants:
    e = L.Engine(num_clients=3, region_bytes=slots * stride, **v)
    mids = [e.register_model(g, P) for g, P in specs]
    for c in range(3):
        _, reg = e.region(c)
        for s in range(slots):
            x = pool[c][s % 8]
            reg[s * stride:s * stride + x.nbytes] = np.frombuffer(x.tobytes(), np.uint8)
    t = traces.arrivals(600, 300.0, seed=3)
    m = traces.model_choices(600, [1, 1, 1], seed=3)
    jct, _ = e.loadgen(t, m, m, np.zeros(600), stride, slots)
    un = {n: round(float(np.median(jct[m == i])) / 1e3, 1) for i, n in enumerate(names)}
    n = 2000
    z = np.zeros(n, dtype=np.int64)
    mm = np.arange(n) % 3
    _, el = e.loadgen(z, mm, mm, z, stride, slots)
    print(json.dumps({"variant": v, "unloaded_p50_us": un, "x_sat": round(n / (el / 1e9), 1)}), flush=True)
    e.shutdown()
