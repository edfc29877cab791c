"""NEXT-3 (P1157-1171, Fig. 14): client CPU cost and JCT of the completion wait.
One client submits ResNet-18 requests open-loop (Poisson) from one thread; a second
thread waits for completions with (a) a spinning poll, (b) PAELLA_HYBRID.  Reports the
waiter's CPU utilisation (thread CPU time / wall) and the client-observed JCT."""
import json
import os
import sys
import threading
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from paper_conf_sosp_ngd023_b200 import _lib as L  # noqa: E402
from workload import archs, rng  # noqa: E402

rate = float(sys.argv[1]) if len(sys.argv) > 1 else 2000.0
n = int(sys.argv[2]) if len(sys.argv) > 2 else 4000
g = archs.build("resnet18")
e = L.Engine(num_clients=1, lookahead=3, slack=1184, launch_threads=4)
mid = e.register_model(g, rng.model_params(g))
info = e.model_info(mid)
need = info["input_bytes"] + info["output_bytes"]
stride = (need + 4095) // 4096 * 4096
_, reg = e.region(0)
x = rng.image(g, 0)
for s in range(64):
    reg[s * stride:s * stride + x.nbytes] = np.frombuffer(x.tobytes(), np.uint8)
out = {}
for label, flags in (("spin", 0), ("hybrid", L.HYBRID)):
    t_sub = {}
    jct = []
    done = [0]

    def waiter():
        t0 = time.thread_time()
        while done[0] < n:
            rid, st = e.poll(0, flags)
            if rid >= 0:
                jct.append(time.perf_counter_ns() - t_sub[rid])
                done[0] += 1
        out[label + "_cpu_s"] = time.thread_time() - t0

    gaps = np.random.default_rng(1).exponential(1.0 / rate, n)
    th = threading.Thread(target=waiter)
    th.start()
    w0 = time.perf_counter()
    due = time.perf_counter()
    for i in range(n):
        due += gaps[i]
        while time.perf_counter() < due:
            pass
        t = time.perf_counter_ns()
        rid = e.submit(0, mid, (i % 64) * stride, need)
        t_sub[rid] = t
    th.join()
    wall = time.perf_counter() - w0
    j = np.array(jct) / 1e3
    out[label] = {"waiter_cpu_util": round(out.pop(label + "_cpu_s") / wall, 3), "jct_mean_us": round(j.mean(), 1),
                  "jct_p99_us": round(float(np.percentile(j, 99)), 1), "req_s": round(n / wall, 1)}
e.shutdown()
print(json.dumps({"model": "resnet18", "offered_req_s": rate, "requests": n, **out}))
