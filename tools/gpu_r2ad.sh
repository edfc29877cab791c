#!/bin/bash
# Light-load gap: does the resident counter-mirror warp alone slow the naive+PDL path?
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
V='[{"naive": true, "instrument": false, "naive_pdl": true, "launch_threads": 4, "dispatcher_cpus": [2]},
 {"slack": 3552, "lookahead": 6, "max_active": 8, "launch_threads": 8, "dispatcher_cpus": [2]}]'
for r in 1 2; do
NREQ=1500 timeout 600 python tools/load_exp.py c3_dispersion 400 "$V" > gpurun_out/mir_off_$r.jsonl 2>/dev/null; echo "off rc=$?"
PAELLA_NAIVE_MIRROR=1 NREQ=1500 timeout 600 python tools/load_exp.py c3_dispersion 400 "$V" > gpurun_out/mir_on_$r.jsonl 2>/dev/null; echo "on rc=$?"
done
for f in gpurun_out/mir_*.jsonl; do echo $f; python -c "
import json,sys
for l in open('$f'):
    d=json.loads(l); print(' ', d['variant'].get('naive',False), d['mean_us'], d['p99_us'], d['per_model_mean_us'])"; done
