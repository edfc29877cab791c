"""Capture target for ncu --profile-from-start off: one isolated run of a model (registered
and warmed unprofiled), between cuProfilerStart/Stop.  Diagnosis tool (no oracle).

    ncu --profile-from-start off -k regex:k_conv_tc --launch-skip 2 --launch-count 1 --set full \\
        --import-source on -o /tmp/l python tools/ncu_one_layer.py densenet121
"""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sosp_ngd023_b200 import _lib as L  # noqa: E402
from workload import archs, rng  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "densenet121"
cuda = ctypes.CDLL("libcuda.so.1")
with L.Engine(num_clients=1) as e:
    g = archs.build(name)
    mid = e.register_model(g, rng.model_params(g), name=name)
    x = rng.image(g, 0)
    e.run_isolated(mid, x)
    cuda.cuProfilerStart()
    e.run_isolated(mid, x)
    cuda.cuProfilerStop()
