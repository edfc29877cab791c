#!/bin/bash
# NEXT-4 branch concurrency with the final configuration (launch-ahead 6 unplaced).
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
V='[{"slack": 3552, "lookahead": 6, "lookahead_unplaced": true, "max_active": 8, "launch_threads": 8, "dispatcher_cpus": [2]},
 {"slack": 3552, "lookahead": 6, "lookahead_unplaced": true, "max_active": 8, "launch_threads": 8, "dispatcher_cpus": [2], "branches": true}]'
for lam in 400 4000 6000; do
n=$([ $lam = 400 ] && echo 1500 || echo 4000)
NREQ=$n timeout 900 python tools/load_exp.py c3_dispersion $lam "$V" > gpurun_out/brn_$lam.jsonl 2>/dev/null; echo "lam $lam rc=$?"
python -c "
import json
for l in open('gpurun_out/brn_$lam.jsonl'):
    d=json.loads(l); print('  $lam', d['variant'].get('branches',False), d['mean_us'], d['p99_us'], d['per_model_mean_us'])"
done
