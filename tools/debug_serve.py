import os, sys, time, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
from paper_conf_sosp_ngd023_b200 import _lib as L
from workload import archs, rng, traces
os.environ["PAELLA_DEBUG"] = "1"
v = json.loads(sys.argv[1])
names = ["resnet18", "mobilenet_v2", "squeezenet1_1"]
specs = [(archs.build(n), None) for n in names]
specs = [(g, rng.model_params(g)) for g, _ in specs]
slots, stride = 128, 1 << 20
e = L.Engine(num_clients=3, region_bytes=slots * stride, **v)
mids = [e.register_model(g, P) for g, P in specs]
for c in range(3):
    _, reg = e.region(c)
    x = rng.image(specs[c][0], 0)
    for s in range(slots):
        reg[s * stride:s * stride + x.nbytes] = np.frombuffer(x.tobytes(), np.uint8)
t = traces.arrivals(300, 300.0, seed=3)
m = traces.model_choices(300, [1, 1, 1], seed=3)
jct, _ = e.loadgen(t, m, m, np.zeros(300), stride, slots)
print("done", np.median(jct) / 1e3, flush=True)
e.shutdown()
