"""Experiment: JCT of serving variants at a fixed offered load, with the dispatcher's
decision diagnostics (why decide() passes stopped, average ready / live jobs, Q).

    python tools/load_exp.py c3_dispersion 3800 '[{"naive": true, "instrument": false}, {"lookahead": 1}]'

Diagnosis tool (no oracle)."""
import json
import os
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import bench  # noqa: E402
from paper_conf_sosp_ngd023_b200 import _lib as L  # noqa: E402
from workload import archs, rng, traces  # noqa: E402

cfgname = sys.argv[1] if len(sys.argv) > 1 else "c2_mix"
lam = float(sys.argv[2]) if len(sys.argv) > 2 else 8000.0
variants = json.loads(sys.argv[3]) if len(sys.argv) > 3 else [{"naive": True, "instrument": False},
                                                               {"lookahead": 1}]
nreq = int(os.environ.get("NREQ", "3000"))
cfg = traces.CONFIGS[cfgname]
names = cfg["models"]
specs = [(archs.build(n), None) for n in names]
specs = [(g, rng.model_params(g)) for g, _ in specs]
pool = [[rng.image(g, i) for i in range(8)] for g, _ in specs]
slots, stride = 128, 1 << 21
if cfg["weights"] is None:   # Fig. 12 convention: inverse of the unloaded job size (fixed estimate)
    est = {"resnet50": 640, "densenet121": 1840, "inception_v3": 1190, "mobilenet_v2": 450}
    cfg = dict(cfg, weights=[1.0 / est[n] for n in names])
for v in variants:
    v = dict(v)
    v.setdefault("launch_threads", 2)
    e = L.Engine(num_clients=len(specs), region_bytes=slots * stride + (1 << 20), max_jobs_per_model=128, **v)
    mids = [e.register_model(g, P) for (g, P) in specs]
    for c, (g, _) in enumerate(specs):
        _, reg = e.region(c)
        for s_ in range(slots):
            x = pool[c][s_ % len(pool[c])]
            reg[s_ * stride:s_ * stride + x.nbytes] = np.frombuffer(x.tobytes(), np.uint8)
    t, mm, ii = bench.make_trace(nreq // 3, lam, cfg, len(names), seed=5)
    e.loadgen(t, mm, mm, ii, stride, slots)   # warm-up
    s0 = e.stats()
    t, mm, ii = bench.make_trace(nreq, lam, cfg, len(names), seed=6)
    jct, el = e.loadgen(t, mm, mm, ii, stride, slots)
    s1 = e.stats()
    st = {k: ([a - b for a, b in zip(s1[k], s0[k])] if isinstance(s1[k], list) else s1[k] - s0[k]) for k in s1}
    dc = max(1, st["decide_calls"])
    res = {"variant": v, "rate": round(nreq / (el / 1e9), 1), "mean_us": round(float(jct.mean()) / 1e3, 1),
           "p50_us": round(float(np.percentile(jct, 50)) / 1e3, 1),
           "p99_us": round(float(np.percentile(jct, 99)) / 1e3, 1),
           "per_model_mean_us": {n: round(float(jct[mm == i].mean()) / 1e3, 1) for i, n in enumerate(names)},
           "stop": st["stop_reason"], "avg_ready": round(st["sum_ready"] / dc, 2),
           "avg_live": round(st["sum_live_jobs"] / dc, 2), "avg_Q": round(st["sum_Q"] / dc, 1),
           "launches": st["launches"], "decides": st["decide_calls"]}
    if st.get("ev_launches"):   # event_time_kind: mean CUDA-event duration of that kernel kind
        res["ev_mean_us"] = round(st["ev_ns"] / st["ev_launches"] / 1e3, 3)
        res["ev_launches"] = st["ev_launches"]
    print(json.dumps(res), flush=True)
    e.shutdown()
