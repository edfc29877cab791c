#!/bin/bash
# Light-load gap: naive+PDL with the instrumented kernels (counter-mode reductions into a
# scratch table) vs plain naive+PDL vs Paella.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
V0='[{"naive": true, "instrument": false, "naive_pdl": true, "launch_threads": 4, "dispatcher_cpus": [2]}]'
V='[{"slack": 3552, "lookahead": 6, "max_active": 8, "launch_threads": 8, "dispatcher_cpus": [2]}]'
for r in 1 2; do
NREQ=1500 timeout 600 python tools/load_exp.py c3_dispersion 400 "$V0" > gpurun_out/ni_plain_$r.jsonl 2>/dev/null
PAELLA_NAIVE_INSTR=1 NREQ=1500 timeout 600 python tools/load_exp.py c3_dispersion 400 "$V0" > gpurun_out/ni_instr_$r.jsonl 2>/dev/null
NREQ=1500 timeout 600 python tools/load_exp.py c3_dispersion 400 "$V" > gpurun_out/ni_paella_$r.jsonl 2>/dev/null
done
for f in gpurun_out/ni_*.jsonl; do python -c "
import json
for l in open('$f'):
    d=json.loads(l); print('$f', d['mean_us'], d['p99_us'], d['per_model_mean_us'])"; done
