#!/bin/bash
# Light-load gap: is logical stream 0 (the policy's favourite) sharing a hardware queue
# with the notification warp's stream (33rd stream, 32 connections)?
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
V='[{"naive": true, "instrument": false, "naive_pdl": true, "launch_threads": 4, "dispatcher_cpus": [2]},
 {"slack": 3552, "lookahead": 6, "max_active": 8, "launch_threads": 8, "dispatcher_cpus": [2]}]'
for rot in 0 16 1; do
PAELLA_STREAM_ROT=$rot NREQ=1500 timeout 600 python tools/load_exp.py c3_dispersion 400 "$V" > gpurun_out/rot_$rot.jsonl 2>/dev/null; echo "rot $rot rc=$?"
python -c "
import json
for l in open('gpurun_out/rot_$rot.jsonl'):
    d=json.loads(l); print('  rot $rot', d['variant'].get('naive',False), d['mean_us'], d['p99_us'], d['per_model_mean_us'])"
done
PAELLA_STREAM_ROT=16 NREQ=3000 timeout 600 python tools/load_exp.py c3_dispersion 4000 "$V" > gpurun_out/rot_load16.jsonl 2>/dev/null
NREQ=3000 timeout 600 python tools/load_exp.py c3_dispersion 4000 "$V" > gpurun_out/rot_load0.jsonl 2>/dev/null
for f in rot_load0 rot_load16; do python -c "
import json
for l in open('gpurun_out/$f.jsonl'):
    d=json.loads(l); print('  $f', d['variant'].get('naive',False), d['mean_us'], d['p99_us'], d['per_model_mean_us'])"; done
