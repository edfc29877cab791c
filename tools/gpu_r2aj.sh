#!/bin/bash
# Light-load gap decomposition: per-job constant vs per-kernel (toy: 4 kernels; C-2 mix).
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
V='[{"naive": true, "instrument": false, "naive_pdl": true, "launch_threads": 4, "dispatcher_cpus": [2]},
 {"slack": 3552, "lookahead": 6, "max_active": 8, "launch_threads": 8, "dispatcher_cpus": [2]}]'
for c in c1_toy c2_mix; do
NREQ=1500 timeout 600 python tools/load_exp.py $c 400 "$V" > gpurun_out/dec_$c.jsonl 2>/dev/null; echo "$c rc=$?"
PAELLA_NAIVE_INSTR=1 NREQ=1500 timeout 600 python tools/load_exp.py $c 400 "$V" > gpurun_out/dec_${c}_ni.jsonl 2>/dev/null
for f in dec_$c dec_${c}_ni; do python -c "
import json
for l in open('gpurun_out/$f.jsonl'):
    d=json.loads(l); print('  $f', d['variant'].get('naive',False), d['mean_us'], d['p50_us'], d['per_model_mean_us'])"; done
done
