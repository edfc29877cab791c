"""Fig. 9 in the simulator (NEXT-2; P1178-1241): throughput and JCT of the C-3 mix as an
injected per-decision scheduler delay grows, with the B200-profiled kernel table of a
bench run (gpurun_out/bench_detail_*.json "kernels": grid, block, regs, smem, T-bar,
instrumented device time) as the synthetic GPU's kernels.  Test-side analysis (it runs
the oracle's simulator); CPU only.

    python tools/sim_delay_sweep.py profiles/r2/bench_detail_r2f.json [n_requests]
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from oracle import sim  # noqa: E402
from workload import traces  # noqa: E402

detail = json.load(open(sys.argv[1]))
n = int(sys.argv[2]) if len(sys.argv) > 2 else 60
names = detail["models"]
models = []
for nm in names:
    ls = []
    for k in detail["kernels"][nm]:
        warps = (k["block"] + 31) // 32
        regs = (k["regs"] * 32 + 255) // 256 * 256 * warps
        smem = (k["smem"] + 1024 + 127) // 128 * 128
        ls.append(sim.Layer(k["grid"], (1, warps, regs, smem, k["tmem"]), int(k["tbar_ns"]), max(1, int(k["instr_ns"]))))
    models.append(ls)
cfg = dict(traces.CONFIGS[detail["config"]], weights=detail["mix_weights"])
lam = detail["lam"]
t = traces.arrivals(n, lam, kind="lognormal", sigma=cfg.get("sigma", 2.0), seed=11)
mm = traces.model_choices(n, cfg["weights"], seed=11)
trace = [(int(t[i]), int(mm[i]), int(mm[i])) for i in range(n)]
rows = []
for dd in (0, 1000, 10000, 50000):
    gpu = sim.GPUModel(launch_delay=3000, notif_delay=5000, decide_delay=dd)
    c = sim.Config(num_clients=len(names), slack=1184, lookahead=3, max_active=8)
    t0 = time.perf_counter()
    r = sim.simulate(c, models, trace, gpu, check=False)
    wall = time.perf_counter() - t0
    jct = np.array(list(r.jct().values())) / 1e3
    span = (max(r.finish.values()) - trace[0][0]) / 1e9
    row = {"decide_delay_ns": dd, "completed": len(r.finish), "throughput_req_s": round(len(r.finish) / span, 1),
           "mean_us": round(float(jct.mean()), 1), "p99_us": round(float(np.percentile(jct, 99)), 1),
           "sim_wall_s": round(wall, 2)}
    rows.append(row)
    print(json.dumps(row), flush=True)
json.dump({"source": sys.argv[1], "lam": lam, "n": n, "rows": rows},
          open(os.path.join("gpurun_out", "sim_delay_sweep.json"), "w"), indent=1)
