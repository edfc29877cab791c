"""B200 rerun of the paper's head-of-line blocking experiment (Fig. 2, P387-445; NEXT-2).

Synthetic jobs (workload.archs.hol_synthetic): a chain of 8 kernels, each ONE block of
128 threads resident for SPIN us (the paper: ~300 us, 9 registers, no shared memory).
Submitting a job's kernels all at once (CUDA-MS, job-by-job) fills the 32 hardware
queues (CUDA_DEVICE_MAX_CONNECTIONS) with dependent kernels: only each queue's head can
run, so at most ~32 one-block kernels run at a time on a GPU that holds 148 x 16 such
blocks.  The dispatcher submits a job's next kernel only once it is runnable (kernel by
kernel, launch-ahead 0, no occupancy cap), onto a large stream pool, so the queues never
hold a blocked kernel in front of a runnable one.

For each system and offered load (open-loop Poisson, 4 clients): goodput (completions/s)
and mean / p99 JCT.  Writes gpurun_out/hol_<tag>.jsonl.

    python tools/hol_exp.py [tag] [spin_us]
"""
import json
import os
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from paper_conf_sosp_ngd023_b200 import _lib as L  # noqa: E402
from workload import archs, rng, traces  # noqa: E402

tag = sys.argv[1] if len(sys.argv) > 1 else "r2"
spin = int(sys.argv[2]) if len(sys.argv) > 2 else 300
g = archs.hol_synthetic(8, spin)
P = rng.model_params(g)
NC = 4
N = int(os.environ.get("NREQ", "3000"))
job_us = 8 * spin
naive_cap = 32 / (job_us * 1e-6)          # closed form: 32 concurrent single-block kernels
rates = [f * naive_cap for f in (0.5, 0.9, 1.5, 3.0, 6.0, 12.0)]
systems = {
    "naive_cuda_ms_32": dict(naive=True, instrument=False, streams=32),
    "naive_cuda_ms_128": dict(naive=True, instrument=False, streams=128),
    "paella_kbk_P32": dict(policy=L.POLICY_FIFO, lookahead=0, slack=1 << 30, streams=32, notify="ring"),
    "paella_kbk_P1024": dict(policy=L.POLICY_FIFO, lookahead=0, slack=1 << 30, streams=1024, notify="ring"),
    "paella_srpt_P1024": dict(policy=L.POLICY_SRPT_DEFICIT, lookahead=0, slack=1 << 30, streams=1024,
                              notify="ring"),
}
out = open(f"gpurun_out/hol_{tag}.jsonl", "w")
print(json.dumps({"spin_us": spin, "kernels_per_job": 8, "naive_bound_jobs_per_s": round(naive_cap, 1)}), flush=True)
for name, kw in systems.items():
    with L.Engine(num_clients=NC, max_jobs_per_model=4096, launch_threads=4, region_bytes=1 << 22,
                  ring_capacity=1 << 16, **kw) as e:
        mid = e.register_model(g, P)
        info = e.model_info(mid)
        stride = (info["input_bytes"] + info["output_bytes"] + 63) // 64 * 64
        slots = 2048
        for c in range(NC):
            _, reg = e.region(c)
            for s in range(slots):
                x = rng.image(g, s % 32)
                reg[s * stride:s * stride + x.nbytes] = np.frombuffer(x.tobytes(), np.uint8)
        for lam in rates:
            t = traces.arrivals(N, lam, kind="poisson", seed=3)
            cl = np.arange(N) % NC
            jct, el = e.loadgen(t, cl, np.zeros(N, dtype=np.int64), np.zeros(N, dtype=np.int64), stride, slots)
            ok = jct >= 0
            row = {"system": name, "offered": round(lam, 1), "goodput": round(ok.sum() / (el / 1e9), 1),
                   "mean_us": round(float(jct[ok].mean()) / 1e3, 1),
                   "p99_us": round(float(np.percentile(jct[ok], 99)) / 1e3, 1),
                   "concurrency": round(float(jct[ok].mean()) / 1e9 * ok.sum() / (el / 1e9), 1)}
            out.write(json.dumps(row) + "\n")
            out.flush()
            print(json.dumps(row), flush=True)
