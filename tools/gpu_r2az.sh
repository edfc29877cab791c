#!/bin/bash
# Job cap admitting in arrival order (cap_fifo) vs SRPT-ordered cap vs FIFO; GPU replay test.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
timeout 900 python -m pytest tests/test_gpu.py -x -q -k "serving_parity_and_replay" > gpurun_out/pytest_r2az.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/pytest_r2az.log
V='[{"naive": true, "instrument": false, "naive_pdl": true, "launch_threads": 4},
 {"max_active": 8},
 {"max_active": 8, "cap_fifo": true},
 {"max_active": 12, "cap_fifo": true},
 {"max_active": 8, "policy": 1}]'
V=$(echo "$V" | python -c "
import json,sys
v=json.load(sys.stdin)
for x in v:
    x.update(dispatcher_cpus=[2])
    if not x.get('naive'): x.update(slack=3552, lookahead=6, lookahead_unplaced=True, launch_threads=8)
print(json.dumps(v))")
for lam in 4000 6000; do
NREQ=4000 timeout 900 python tools/load_exp.py c3_dispersion $lam "$V" > gpurun_out/cf_$lam.jsonl 2>/dev/null; echo "lam $lam rc=$?"
python -c "
import json
for l in open('gpurun_out/cf_$lam.jsonl'):
    d=json.loads(l); v=d['variant']; print('  $lam', {k: v[k] for k in v if k in ('naive','max_active','cap_fifo','policy')}, d['mean_us'], d['p99_us'], d['per_model_mean_us'])"
done
