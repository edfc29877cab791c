"""Config 5 microbenchmarks + device-only kernel timing (no oracle involved)."""
import sys, os, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
from paper_conf_sosp_ngd023_b200 import _lib as L
from workload import archs, rng

e = L.Engine(num_clients=1)
res = {}
for grid in (1, 16, 148, 160, 1184, 4736):
    for G in (16, 1):
        a = e.bench_empty(grid, 128, True, G, 2000)
        b = e.bench_empty(grid, 128, False, G, 2000)
        print(f"empty grid={grid:5d} G={G:2d} instr {a/1e3:7.2f}us plain {b/1e3:7.2f}us  delta {(a-b)/1e3:6.2f}us", flush=True)
p, c = e.bench_roundtrip(2000)
print("roundtrip place p50/p99 %.2f/%.2f us complete p50/p99 %.2f/%.2f us" % (
    np.percentile(p, 50)/1e3, np.percentile(p, 99)/1e3, np.percentile(c, 50)/1e3, np.percentile(c, 99)/1e3))
for name in sys.argv[1:] or ["toy", "resnet18"]:
    g = archs.build(name)
    mid = e.register_model(g, rng.model_params(g))
    ks = e.kernels(mid)
    ti = e.time_kernels(mid, True, 50)
    tp = e.time_kernels(mid, False, 50)
    print(f"{name}: sum instr {ti.sum()/1e3:.1f}us plain {tp.sum()/1e3:.1f}us")
    for i, k in enumerate(ks):
        print(f"   {i:3d} {k['name']:13s} grid {k['grid']:5d} instr {ti[i]/1e3:7.2f}us plain {tp[i]/1e3:7.2f}us  "
              f"{k['bytes']/max(tp[i],1):7.1f} GB/s  {k['flops']/max(tp[i],1)/1e3:7.2f} TF/s")
e.shutdown()
