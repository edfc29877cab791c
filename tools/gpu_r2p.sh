#!/bin/bash
# Sweep: slack B x launch-ahead x job cap K (SRPT), plus FIFO at the best guesses; three loads.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
V='[{"naive": true, "instrument": false, "naive_pdl": true},
 {"slack": 2368, "lookahead": 6, "max_active": 8},
 {"slack": 3552, "lookahead": 6, "max_active": 8},
 {"slack": 4736, "lookahead": 6, "max_active": 8},
 {"slack": 2368, "lookahead": 4, "max_active": 8},
 {"slack": 3552, "lookahead": 4, "max_active": 8},
 {"slack": 3552, "lookahead": 6, "max_active": 6},
 {"slack": 3552, "lookahead": 6, "max_active": 12},
 {"slack": 3552, "lookahead": 6, "max_active": 8, "policy": 1},
 {"slack": 3552, "lookahead": 6, "max_active": 8, "theta": 300}]'
V=$(echo "$V" | python -c "import json,sys; v=json.load(sys.stdin); [x.update(launch_threads=4, dispatcher_cpus=[2]) for x in v]; print(json.dumps(v))")
NREQ=1500 timeout 900 python tools/load_exp.py c3_dispersion 400 "$V" > gpurun_out/sw_light_r2p.jsonl 2> gpurun_out/sw_light_r2p.err; echo "light rc=$?"
NREQ=4000 timeout 900 python tools/load_exp.py c3_dispersion 4000 "$V" > gpurun_out/sw_load_r2p.jsonl 2> gpurun_out/sw_load_r2p.err; echo "load rc=$?"
NREQ=4000 timeout 900 python tools/load_exp.py c3_dispersion 5500 "$V" > gpurun_out/sw_high_r2p.jsonl 2> gpurun_out/sw_high_r2p.err; echo "high rc=$?"
python - <<'PY'
import json
for f in ["gpurun_out/sw_light_r2p.jsonl", "gpurun_out/sw_load_r2p.jsonl", "gpurun_out/sw_high_r2p.jsonl"]:
    print(f)
    for l in open(f):
        d = json.loads(l); v = d["variant"]
        print({k: v[k] for k in v if k not in ("launch_threads", "dispatcher_cpus")}, d["rate"], d["mean_us"], d["p99_us"], d["per_model_mean_us"], d["stop"], d["avg_Q"])
PY
