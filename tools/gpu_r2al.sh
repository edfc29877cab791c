#!/bin/bash
# Light-load gap: do host launches during execution slow running kernel chains?
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
V='[{"naive": true, "instrument": false, "naive_pdl": true, "launch_threads": 4, "dispatcher_cpus": [2]}]'
for n in off 20 5; do
  if [ $n = off ]; then E=X; else E=PAELLA_LAUNCH_NOISE_US; fi
  env $E=$n NREQ=1500 timeout 600 python tools/load_exp.py c3_dispersion 400 "$V" > gpurun_out/noise_$n.jsonl 2>/dev/null; echo "noise $n rc=$?"
  python -c "
import json
for l in open('gpurun_out/noise_$n.jsonl'):
    d=json.loads(l); print('  noise $n', d['mean_us'], d['p99_us'], d['per_model_mean_us'])"
done
