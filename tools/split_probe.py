"""Debug: one conv layer's phase trace under forced split factors / reductions (split
cache), e.g. python tools/split_probe.py densenet121 4 "1 0" "2 0" "2 1" "4 0".
Diagnosis tool (no oracle)."""
import os
import sys
import tempfile

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sosp_ngd023_b200 import _lib as L  # noqa: E402
from workload import archs, rng  # noqa: E402

name, layer = sys.argv[1], int(sys.argv[2])
e = L.Engine(num_clients=1)
g = archs.build(name)
P = rng.model_params(g)
x = rng.image(g, 0)
for spec in sys.argv[3:]:
    sp, dsm = (int(v) for v in spec.split())
    mname = f"{name}-p{sp}-{dsm}"
    f = tempfile.NamedTemporaryFile("w", suffix=".txt", delete=False)
    f.write(f"{mname} {layer} {sp} {dsm}\n")
    f.close()
    os.environ["PAELLA_SPLITS_FILE"] = f.name
    mid = e.register_model(g, P, name=mname)
    del os.environ["PAELLA_SPLITS_FILE"]
    ks = e.kernels(mid)
    tt = e.time_kernels(mid, instrumented=True, reps=100)
    print(f"{name} layer {layer} split {sp} dsmem {dsm}: grid {ks[layer]['grid']} time_kernels {tt[layer]} ns",
          flush=True)
    os.environ["PAELLA_TRACE_KERNEL"] = str(layer)
    for _ in range(2):
        e.run_isolated(mid, x, timing=True)
    sys.stderr.flush()
    del os.environ["PAELLA_TRACE_KERNEL"]
e.shutdown()
