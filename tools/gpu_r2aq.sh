#!/bin/bash
# Are bursts of host launches cheaper for a running chain than the same launches spread out?
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
V='[{"naive": true, "instrument": false, "naive_pdl": true, "launch_threads": 4, "dispatcher_cpus": [2]}]'
for cfg in off:0:1 p5:5:1 p20b4:20:4 p40b8:40:8; do
  n=$(echo $cfg | cut -d: -f1); us=$(echo $cfg | cut -d: -f2); b=$(echo $cfg | cut -d: -f3)
  if [ $n = off ]; then E=X; else E=PAELLA_LAUNCH_NOISE_US; fi
  env $E=$us PAELLA_LAUNCH_NOISE_BURST=$b NREQ=1500 timeout 600 python tools/load_exp.py c3_dispersion 400 "$V" > gpurun_out/burst_$n.jsonl 2>/dev/null
  python -c "
import json
for l in open('gpurun_out/burst_$n.jsonl'):
    d=json.loads(l); print('  $n', d['mean_us'], d['p99_us'], d['per_model_mean_us'])"
done
