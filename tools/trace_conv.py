"""Debug: per-CTA phase timestamps of tcgen05 conv kernels (PAELLA_TRACE_KERNEL)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sosp_ngd023_b200 import _lib as L
from workload import archs, rng
name = sys.argv[1]; ks = [int(x) for x in sys.argv[2:]]
e = L.Engine(num_clients=1)
g = archs.build(name); mid = e.register_model(g, rng.model_params(g))
x = rng.image(g, 0)
for k in ks:
    os.environ["PAELLA_TRACE_KERNEL"] = str(k)
    for _ in range(3):
        e.run_isolated(mid, x, timing=True)
e.shutdown()
