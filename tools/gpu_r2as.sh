#!/bin/bash
# Final-config neighbourhood (launch-ahead 6 unplaced): K, B, theta at moderate / high load.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
V='[{"naive": true, "instrument": false, "naive_pdl": true, "launch_threads": 4},
 {"slack": 3552, "max_active": 8},
 {"slack": 3552, "max_active": 6},
 {"slack": 3552, "max_active": 12},
 {"slack": 4736, "max_active": 8},
 {"slack": 3552, "max_active": 8, "theta": 30},
 {"slack": 3552, "max_active": 8, "theta": 300},
 {"slack": 3552, "max_active": 0}]'
V=$(echo "$V" | python -c "
import json,sys
v=json.load(sys.stdin)
for x in v:
    x.update(dispatcher_cpus=[2])
    if not x.get('naive'): x.update(lookahead=6, lookahead_unplaced=True, launch_threads=8)
print(json.dumps(v))")
for lam in 4000 6000; do
NREQ=4000 timeout 900 python tools/load_exp.py c3_dispersion $lam "$V" > gpurun_out/nb_$lam.jsonl 2> gpurun_out/nb_$lam.err; echo "lam $lam rc=$?"
python - $lam <<'PY'
import json, sys
for l in open(f"gpurun_out/nb_{sys.argv[1]}.jsonl"):
    d = json.loads(l); v = d["variant"]
    print({k: v[k] for k in v if k not in ("dispatcher_cpus", "lookahead", "lookahead_unplaced", "launch_threads")}, d["mean_us"], d["p99_us"], d["per_model_mean_us"])
PY
done
