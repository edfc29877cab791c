"""Capture target for `ncu --profile-from-start off`: registers the models of a bench
config (split-K autotuning and T-bar profiling run unprofiled), then runs ONE isolated
request of each model between cudaProfilerStart/Stop, so the capture holds exactly the
served kernel configuration of one request per model.  No oracle involved."""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sosp_ngd023_b200 import _lib as L  # noqa: E402
from workload import archs, rng, traces  # noqa: E402

cfg = traces.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "c2_mix"]
e = L.Engine(num_clients=1)
mids = []
for nm in cfg["models"]:
    g = archs.build(nm)
    mids.append((e.register_model(g, rng.model_params(g), name=nm), g))
for mid, g in mids:   # warm (unprofiled)
    e.run_isolated(mid, rng.image(g, 0))
cuda = ctypes.CDLL("libcuda.so.1")
ctx = ctypes.c_void_p()
cuda.cuDevicePrimaryCtxRetain(ctypes.byref(ctx), 0)
cuda.cuCtxPushCurrent(ctx)
assert cuda.cuProfilerStart() == 0
for mid, g in mids:
    e.run_isolated(mid, rng.image(g, 0))
assert cuda.cuProfilerStop() == 0
e.shutdown()
print("captured one request of", cfg["models"])
