"""Per-kind instrumentation slowdown from gpurun_out/kernel_times*.json (diagnosis)."""
import json
import sys

import numpy as np

d = json.load(open(sys.argv[1]))
rows = [(m, r) for m, rs in d["models"].items() for r in rs]
by = {}
for m, r in rows:
    s = r["t_instr_ns"] / max(1, r["t_plain_ns"]) - 1
    by.setdefault(r["name"], []).append((s, r["t_plain_ns"], m, r["i"]))
for k, v in sorted(by.items()):
    s = np.array([x[0] for x in v])
    t = np.array([x[1] for x in v])
    print(f"{k:16s} n={len(v):3d} median {np.median(s)*100:5.1f}% p90 {np.percentile(s,90)*100:5.1f}% "
          f"max {s.max()*100:5.1f}%  mean t {t.mean()/1e3:.2f}us  abs delta med {np.median(s*t)/1e3:.2f}us")
allv = np.array([x[0] for v in by.values() for x in v])
print(f"ALL n={len(allv)} median {np.median(allv)*100:.1f}% p90 {np.percentile(allv,90)*100:.1f}% max {allv.max()*100:.1f}%")
for s, x in sorted([(x[0], x) for v in by.values() for x in v])[-8:]:
    print(f"  {x[2]:14s} #{x[3]:3d} +{s*100:.1f}% plain {x[1]/1e3:.2f}us")
