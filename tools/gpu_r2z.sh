#!/bin/bash
# Launcher threads and job cap at high load (C-3): does the host launch path bound X_sat?
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
V='[{"naive": true, "instrument": false, "naive_pdl": true, "launch_threads": 4},
 {"slack": 3552, "lookahead": 6, "max_active": 8, "launch_threads": 4},
 {"slack": 3552, "lookahead": 6, "max_active": 8, "launch_threads": 8},
 {"slack": 3552, "lookahead": 6, "max_active": 12, "launch_threads": 8},
 {"slack": 3552, "lookahead": 6, "max_active": 8, "launch_threads": 8, "policy": 1},
 {"slack": 3552, "lookahead": 6, "max_active": 12, "launch_threads": 8, "policy": 1},
 {"naive": true, "instrument": false, "naive_pdl": true, "launch_threads": 8}]'
V=$(echo "$V" | python -c "import json,sys; v=json.load(sys.stdin); [x.update(dispatcher_cpus=[2]) for x in v]; print(json.dumps(v))")
for lam in 4000 6000 7500; do
NREQ=4000 timeout 900 python tools/load_exp.py c3_dispersion $lam "$V" > gpurun_out/lt_$lam.jsonl 2> gpurun_out/lt_$lam.err; echo "lam $lam rc=$?"
python - $lam <<'PY'
import json, sys
for l in open(f"gpurun_out/lt_{sys.argv[1]}.jsonl"):
    d = json.loads(l); v = d["variant"]
    print({k: v[k] for k in v if k not in ("dispatcher_cpus",)}, d["rate"], d["mean_us"], d["p99_us"], d["stop"], d["avg_Q"])
PY
done
