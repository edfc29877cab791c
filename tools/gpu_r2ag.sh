#!/bin/bash
# Light-load gap: Paella variants (launch path).
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
V='[{"slack": 3552, "lookahead": 6, "max_active": 8, "launch_threads": 8, "dispatcher_cpus": [2]},
 {"slack": 3552, "lookahead": 6, "max_active": 8, "launch_threads": 0, "dispatcher_cpus": [2]},
 {"slack": 3552, "lookahead": 6, "max_active": 8, "launch_threads": 1, "dispatcher_cpus": [2]},
 {"slack": 3552, "lookahead": 7, "max_active": 8, "launch_threads": 8, "dispatcher_cpus": [2], "streams": 16},
 {"slack": 3552, "lookahead": 6, "max_active": 8, "launch_threads": 8, "dispatcher_cpus": [2], "group": 1}]'
NREQ=1500 timeout 900 python tools/load_exp.py c3_dispersion 400 "$V" > gpurun_out/lp.jsonl 2>gpurun_out/lp.err; echo "rc=$?"
python -c "
import json
for l in open('gpurun_out/lp.jsonl'):
    d=json.loads(l); v=d['variant']; print({k: v[k] for k in v if k not in ('dispatcher_cpus','slack','max_active')}, d['mean_us'], d['p99_us'], d['per_model_mean_us'])"
tail -2 gpurun_out/lp.err
