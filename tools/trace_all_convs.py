"""Debug: per-CTA phase timestamps (PAELLA_TRACE_KERNEL) of EVERY tcgen05 conv of the
given models, each inside an isolated PDL chain (gate-released, as in time_kernels).
The phase table goes to stderr (one block per traced kernel); the layer table (index,
grid, smem, flops, bytes) to stdout as JSON lines.  Summarise with
tools/trace_summary.py.  Diagnosis tool (no oracle)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sosp_ngd023_b200 import _lib as L  # noqa: E402
from workload import archs, rng  # noqa: E402

names = sys.argv[1:] or ["resnet50"]
e = L.Engine(num_clients=1)
for name in names:
    g = archs.build(name)
    mid = e.register_model(g, rng.model_params(g), name=name)
    x = rng.image(g, 0)
    ks = e.kernels(mid)
    for k, info in enumerate(ks):
        if not info["name"].startswith("conv_tcgen05"):
            continue
        os.environ["PAELLA_TRACE_KERNEL"] = str(k)
        for _ in range(2):
            e.run_isolated(mid, x, timing=True)
        sys.stderr.flush()
        print(json.dumps(dict(model=name, k=k, grid=info["grid"], smem=info["smem"], flops=int(info["flops"]),
                              bytes=int(info["bytes"]), tbar_ns=int(info["tbar_ns"]))), flush=True)
    os.environ.pop("PAELLA_TRACE_KERNEL", None)
e.shutdown()
