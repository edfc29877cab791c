#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
V='[{"naive": true, "instrument": false, "naive_pdl": true, "launch_threads": 4, "dispatcher_cpus": [2]},
 {"slack": 3552, "lookahead": 6, "max_active": 8, "launch_threads": 8, "dispatcher_cpus": [2]}]'
PAELLA_LAUNCH_STATS=1 NREQ=1500 timeout 600 python tools/load_exp.py c3_dispersion 400 "$V" > gpurun_out/ls_light.jsonl 2> gpurun_out/ls_light.err; echo "rc=$?"
PAELLA_LAUNCH_STATS=1 NREQ=3000 timeout 600 python tools/load_exp.py c3_dispersion 4000 "$V" > gpurun_out/ls_load.jsonl 2> gpurun_out/ls_load.err; echo "rc=$?"
for f in light load; do echo == $f; grep "\[paella\]" gpurun_out/ls_$f.err; cut -c1-200 gpurun_out/ls_$f.jsonl; done
