#!/bin/bash
# Light-load gap: does the mirror's polling of the counter lines slow the kernels (L2
# contention with the blocks' count reductions)?  Mirror pacing 0 / 500 / 2000 ns.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
V0='[{"naive": true, "instrument": false, "naive_pdl": true, "launch_threads": 4, "dispatcher_cpus": [2]}]'
V='[{"slack": 3552, "lookahead": 6, "max_active": 8, "launch_threads": 8, "dispatcher_cpus": [2]}]'
NREQ=1500 timeout 600 python tools/load_exp.py c3_dispersion 400 "$V0" > gpurun_out/pace_naive.jsonl 2>/dev/null
for p in 0 500 2000 0; do
PAELLA_MIRROR_PACE_NS=$p NREQ=1500 timeout 600 python tools/load_exp.py c3_dispersion 400 "$V" > gpurun_out/pace_$p.jsonl 2>/dev/null; echo "pace $p rc=$?"
python -c "
import json
for l in open('gpurun_out/pace_$p.jsonl'):
    d=json.loads(l); print('  pace $p', d['mean_us'], d['p99_us'], d['per_model_mean_us'])"
done
python -c "
import json
for l in open('gpurun_out/pace_naive.jsonl'):
    d=json.loads(l); print('  naive_pdl', d['mean_us'], d['p99_us'], d['per_model_mean_us'])"
