#!/bin/bash
# NEXT-1 variant: launch-ahead without the placement test, light / moderate / high load.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
V='[{"naive": true, "instrument": false, "naive_pdl": true, "launch_threads": 4},
 {"slack": 3552, "lookahead": 6, "max_active": 8, "launch_threads": 8},
 {"slack": 3552, "lookahead": 6, "max_active": 8, "launch_threads": 8, "lookahead_unplaced": true},
 {"slack": 3552, "lookahead": 4, "max_active": 8, "launch_threads": 8, "lookahead_unplaced": true},
 {"slack": 3552, "lookahead": 3, "max_active": 8, "launch_threads": 8, "lookahead_unplaced": true},
 {"slack": 4736, "lookahead": 6, "max_active": 8, "launch_threads": 8, "lookahead_unplaced": true},
 {"slack": 3552, "lookahead": 6, "max_active": 8, "launch_threads": 8, "lookahead_unplaced": true, "policy": 1}]'
V=$(echo "$V" | python -c "import json,sys; v=json.load(sys.stdin); [x.update(dispatcher_cpus=[2]) for x in v]; print(json.dumps(v))")
for lam in 400 4000 6000; do
n=$([ $lam = 400 ] && echo 1500 || echo 4000)
NREQ=$n timeout 900 python tools/load_exp.py c3_dispersion $lam "$V" > gpurun_out/un_$lam.jsonl 2> gpurun_out/un_$lam.err; echo "lam $lam rc=$?"
python - $lam <<'PY'
import json, sys
for l in open(f"gpurun_out/un_{sys.argv[1]}.jsonl"):
    d = json.loads(l); v = d["variant"]
    print({k: v[k] for k in v if k not in ("dispatcher_cpus", "max_active")}, d["mean_us"], d["p99_us"], d["per_model_mean_us"], d["stop"])
PY
done
V2='[{"naive": true, "instrument": false, "naive_pdl": true, "launch_threads": 4, "dispatcher_cpus": [2]},
 {"slack": 3552, "lookahead": 6, "max_active": 8, "launch_threads": 8, "dispatcher_cpus": [2]},
 {"slack": 3552, "lookahead": 6, "max_active": 8, "launch_threads": 8, "dispatcher_cpus": [2], "lookahead_unplaced": true}]'
for c in c1_toy c2_mix; do
NREQ=1500 timeout 600 python tools/load_exp.py $c 400 "$V2" > gpurun_out/un_$c.jsonl 2>/dev/null
python -c "
import json
for l in open('gpurun_out/un_$c.jsonl'):
    d=json.loads(l); v=d['variant']; print('$c', v.get('naive',False), v.get('lookahead_unplaced',False), d['mean_us'], d['p99_us'], d['per_model_mean_us'])"
done
