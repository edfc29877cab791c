import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sosp_ngd023_b200 import _lib as L
e = L.Engine(num_clients=1)
for dev in (0, 1):
    if not dev: os.environ["PAELLA_BENCH_DIRECT"] = "1"
    else: os.environ.pop("PAELLA_BENCH_DIRECT", None)
    for grid in (1, 16, 148, 1184):
        a = e.bench_empty(grid, 128, True, 16, 1000)
        b = e.bench_empty(grid, 128, False, 16, 1000)
        print(f"devring={dev} grid={grid:5d} instr {a/1e3:6.2f} plain {b/1e3:6.2f} delta {(a-b)/1e3:6.2f}", flush=True)
e.shutdown()
