"""Config 5 (BASELINE configs[4]; P1881-1897, Fig. 15): instrumentation overhead and
notification latency, written to gpurun_out/c5_<tag>.json and printed as a table.

(i)   empty kernel, grids {16, 148, 160, 1184, 4736} x 128 threads, 2,000 launches each
      (the paper used 16 / 160 blocks), instrumented vs the uninstrumented twin, for the
      three notification paths: counter mode (served default), the device ring with the
      forwarding warp at G = 1 and G = 16, and the paper's direct ring write at G = 16;
(ii)  ring round trip of a 1-block kernel (launch -> PLACEMENT / COMPLETION visible to
      the host), 10,000 samples, p50 / p99;
(iii) dispatcher launches/s and records/s per core come from the bench detail file.

    python tools/c5_table.py [tag]
"""
import json
import os
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from paper_conf_sosp_ngd023_b200 import _lib as L  # noqa: E402

tag = sys.argv[1] if len(sys.argv) > 1 else "r2"
GRIDS = (16, 148, 160, 1184, 4736)
out = {"empty_us": {}, "roundtrip_us": None}
for label, kw, G in (("counters", dict(notify="counters"), 16), ("ring_G1", dict(notify="ring"), 1),
                     ("ring_G16", dict(notify="ring"), 16), ("direct_G16", dict(notify="direct"), 16)):
    if label.startswith("direct"):
        os.environ["PAELLA_BENCH_DIRECT"] = "1"    # records straight into the pinned host ring
    else:
        os.environ.pop("PAELLA_BENCH_DIRECT", None)
    with L.Engine(num_clients=1, **kw) as e:
        rows = {}
        for grid in GRIDS:
            a = e.bench_empty(grid, 128, True, G, 2000)
            b = e.bench_empty(grid, 128, False, G, 2000)
            rows[grid] = {"instr": round(a / 1e3, 3), "plain": round(b / 1e3, 3), "delta": round((a - b) / 1e3, 3)}
            print(f"{label:10s} grid {grid:5d}: instr {a/1e3:7.3f} us plain {b/1e3:7.3f} us delta {(a-b)/1e3:6.3f} us",
                  flush=True)
        out["empty_us"][label] = rows
        if label == "counters":
            p, c = e.bench_roundtrip(10000)
            out["roundtrip_us"] = {q: round(float(np.percentile(x, pc)) / 1e3, 3)
                                   for q, x, pc in (("placement_p50", p, 50), ("placement_p99", p, 99),
                                                    ("completion_p50", c, 50), ("completion_p99", c, 99))}
            print("round trip (us):", out["roundtrip_us"], flush=True)
os.makedirs("gpurun_out", exist_ok=True)
json.dump(out, open(f"gpurun_out/c5_{tag}.json", "w"), indent=1)
