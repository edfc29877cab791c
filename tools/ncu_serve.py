"""Capture target for `ncu --profile-from-start off`: the C-3 mix served by the Paella arm
(bench configuration) and by the naive arm -- models registered and warmed unprofiled,
then a short open-loop trace of each system between cuProfilerStart/Stop, so the launch
list holds the kernels exactly as served (shares of device time).  No oracle involved.

    python tools/ncu_serve.py [n_requests] [rate]
"""
import ctypes
import os
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import bench  # noqa: E402
from paper_conf_sosp_ngd023_b200 import _lib as L  # noqa: E402
from workload import archs, rng, traces  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 150
rate = float(sys.argv[2]) if len(sys.argv) > 2 else 3500.0
cfg = dict(traces.CONFIGS["c3_dispersion"], weights=[1 / 535, 1 / 1179, 1 / 997, 1 / 389])
names = cfg["models"]
specs = [(archs.build(nm), None) for nm in names]
specs = [(g, rng.model_params(g)) for g, _ in specs]
pool = [[rng.image(g, i) for i in range(4)] for g, _ in specs]
sizes = [int(np.prod(g.nodes[0]["out"])) * 4 + g.num_classes * 4 for (g, _) in specs]
stride = (max(sizes) + 4095) // 4096 * 4096
slots = 64
region = slots * stride + (1 << 20)
cuda = ctypes.CDLL("libcuda.so.1")
t, mm, ii = bench.make_trace(n, rate, cfg, len(names), seed=77)
for label, kw in (("paella", dict(policy=L.POLICY_SRPT_DEFICIT, slack=3552, lookahead=6, max_active=8, launch_threads=8,
                                lookahead_unplaced=True)),
                  ("naive", dict(naive=True, instrument=False))):
    a = bench.Arm(L, label, specs, pool, 1, region, stride, slots, False,
                  **dict(dict(launch_threads=4, max_jobs_per_model=64), **kw))
    a.serve(*bench.make_trace(40, rate, cfg, len(names), seed=5))   # warm, unprofiled
    ctx = ctypes.c_void_p()
    cuda.cuDevicePrimaryCtxRetain(ctypes.byref(ctx), 0)
    cuda.cuCtxPushCurrent(ctx)
    assert cuda.cuProfilerStart() == 0
    a.serve(t, mm, ii)
    assert cuda.cuProfilerStop() == 0
    a.close()
    print("served", n, "requests:", label, flush=True)
