"""C-3 load sweep: every arm built once, then served at
rho in {0.5 .. 0.9} x X_sat,1(naive) (bisection, per config) with 3 trace seeds, for the
bursty C-3 mix and its variants (sigma = 1.5, uniform mix).  Writes JSONL rows
{config, rho, seed, arm, mean/p50/p99 per model and mix} to gpurun_out/rho_sweep_<tag>.jsonl.

    python tools/rho_sweep.py [tag] [configs comma-separated]
"""
import json
import os
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import bench  # noqa: E402
from paper_conf_sosp_ngd023_b200 import _lib as L  # noqa: E402
from workload import archs, rng, traces  # noqa: E402

tag = sys.argv[1] if len(sys.argv) > 1 else "r2"
cfgs = (sys.argv[2] if len(sys.argv) > 2 else "c3_dispersion,c3_sigma15,c3_uniform").split(",")
RHOS = [float(x) for x in os.environ.get("RHOS", "0.5,0.6,0.7,0.8,0.9").split(",")]
SEEDS = [int(x) for x in os.environ.get("SEEDS", "1,2,3").split(",")]
NREQ = int(os.environ.get("NREQ", "2000"))
names = traces.CONFIGS["c3_dispersion"]["models"]
specs = [(archs.build(n), None) for n in names]
specs = [(g, rng.model_params(g)) for g, _ in specs]
pool = [[rng.image(g, i) for i in range(32)] for g, _ in specs]
sizes = [int(np.prod(g.nodes[0]["out"])) * 4 + g.num_classes * 4 for (g, _) in specs]
stride = (max(sizes) + 4095) // 4096 * 4096
slots = 256
region = slots * stride + (1 << 20)
common = dict(max_jobs_per_model=128, dispatcher_cpus=[2])
# the bench's arm configurations (bench.py defaults: each arm with its best launcher count)
arms = {
    "naive": dict(naive=True, instrument=False, launch_threads=4),
    "naive_pdl": dict(naive=True, instrument=False, naive_pdl=True, launch_threads=4),
    "paella": dict(policy=L.POLICY_SRPT_DEFICIT, theta=100, slack=3552, lookahead=6, max_active=8, launch_threads=8,
                   lookahead_unplaced=True),
    "paella_fifo": dict(policy=L.POLICY_FIFO, slack=3552, lookahead=6, max_active=8, launch_threads=8,
                        lookahead_unplaced=True),
}
out = open(f"gpurun_out/rho_sweep_{tag}.jsonl", "w")
# calibration per config on the naive arm: unloaded medians (mix weights), X_sat bisection
a = bench.Arm(L, "naive", specs, pool, 1, region, stride, slots, False, **common, **arms["naive"])
cal = {}
x0 = bench.closed_burst(a, len(names), 1500)
for cn in cfgs:
    cfg = dict(traces.CONFIGS[cn])
    t1, m1, i1 = bench.make_trace(300, 200.0, cfg, len(names), seed=7)
    j1, _ = a.serve(t1, m1, i1)
    med = [float(np.median(j1[m1 == m])) / 1e3 for m in range(len(names))]
    if cfg["weights"] is None:
        cfg["weights"] = [1.0 / x for x in med]
    xs = bench.saturation(a, cfg, len(names), 3000, x0, iters=5)
    cal[cn] = (cfg, xs)
    print(json.dumps({"config": cn, "x_sat_naive": round(xs, 1), "unloaded_p50_us": med}), flush=True)
    out.write(json.dumps({"config": cn, "x_sat_naive": xs, "unloaded_p50_us": med}) + "\n")
a.close()
for arm, kw in arms.items():
    a = bench.Arm(L, arm, specs, pool, 1, region, stride, slots, False, **common, **kw)
    for cn in cfgs:
        cfg, xs = cal[cn]
        for rho in RHOS:
            for seed in SEEDS:
                t, mm, ii = bench.make_trace(NREQ, rho * xs, cfg, len(names), seed=5000 + 97 * seed)
                a.serve(*bench.make_trace(300, rho * xs, cfg, len(names), seed=9000 + seed))   # warm
                jct, el = a.serve(t, mm, ii)
                st = bench.jct_stats(jct, mm, names)
                row = {"config": cn, "rho": rho, "seed": seed, "arm": arm, "lam": round(rho * xs, 1),
                       "served": round((jct >= 0).sum() / (el / 1e9), 1), "jct": st}
                out.write(json.dumps(row) + "\n")
                out.flush()
                print(cn, rho, seed, arm, round(st["mix"]["mean_us"]), round(st["mix"]["p99_us"]), flush=True)
    a.close()
