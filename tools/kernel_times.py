"""Per-kernel isolated device times of every model (back-to-back launches of the same
kernel on one stream behind a gate, CUDA events), with the algorithmic bytes/flops of
each launch, uninstrumented and instrumented.  Writes gpurun_out/kernel_times.json
and prints a per-model summary.  Diagnosis tool (no oracle)."""
import json
import os
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from paper_conf_sosp_ngd023_b200 import _lib as L  # noqa: E402
from workload import archs, rng  # noqa: E402

names = sys.argv[1:] or ["resnet18", "mobilenet_v2", "squeezenet1_1", "resnet50", "densenet121", "inception_v3"]
out = {}
with L.Engine(num_clients=1) as e:
    empty = {g: e.bench_empty(g, instrumented=False) for g in (1, 16, 148)}
    print("empty kernel ns/launch:", {k: round(v, 1) for k, v in empty.items()})
    for name in names:
        g = archs.build(name)
        mid = e.register_model(g, rng.model_params(g), name=name)
        ks = e.kernels(mid)
        tp = e.time_kernels(mid, instrumented=False, reps=100)
        ti = e.time_kernels(mid, instrumented=True, reps=100)
        rows = []
        for i, k in enumerate(ks):
            rows.append(dict(i=i, name=k["name"], grid=k["grid"], block=k["block"], regs=k["regs"],
                             smem=k["smem"], flops=int(k["flops"]), bytes=int(k["bytes"]),
                             t_plain_ns=int(tp[i]), t_instr_ns=int(ti[i])))
        out[name] = rows
        by = {}
        for r in rows:
            b = by.setdefault(r["name"], [0, 0, 0, 0])
            b[0] += 1
            b[1] += r["t_plain_ns"]
            b[2] += r["t_instr_ns"]
            b[3] += r["bytes"]
        print(f"{name}: {len(rows)} kernels, sum plain {tp.sum()/1e3:.1f} us, instr {ti.sum()/1e3:.1f} us")
        for k, (n, a, b, by_) in sorted(by.items(), key=lambda kv: -kv[1][1]):
            print(f"   {k:14s} n={n:3d} plain {a/1e3:7.1f} us instr {b/1e3:7.1f} us  "
                  f"mean {a/n/1e3:5.2f} us  {by_/max(a,1):6.1f} GB/s")
        top = sorted(rows, key=lambda r: -r["t_plain_ns"])[:6]
        for r in top:
            print(f"     #{r['i']:3d} {r['name']:10s} g={r['grid']:4d} {r['t_plain_ns']/1e3:6.2f} us "
                  f"{r['bytes']/1e6:6.2f} MB {r['flops']/1e9:6.3f} GF")
# config 5 (BASELINE): per-kernel instrumentation slowdown over every distinct layer
# kernel of the models above (instrumented as served vs the uninstrumented twin)
sl = np.array([r["t_instr_ns"] / max(1, r["t_plain_ns"]) - 1.0 for rows in out.values() for r in rows])
print(f"per-kernel instrumentation slowdown over {len(sl)} kernels: median {np.median(sl)*100:.1f} %, "
      f"p90 {np.percentile(sl, 90)*100:.1f} %, max {sl.max()*100:.1f} %")
os.makedirs("gpurun_out", exist_ok=True)
json.dump({"empty_ns": empty, "models": out}, open("gpurun_out/kernel_times.json", "w"))
