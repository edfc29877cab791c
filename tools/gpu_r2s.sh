#!/bin/bash
# Served conv duration (CUDA events around every tcgen05 conv launch, dispatcher launches
# itself): naive+PDL vs Paella at light load and under load.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
V='[{"naive": true, "instrument": false, "naive_pdl": true},
 {"slack": 3552, "lookahead": 6, "max_active": 8},
 {"naive": true, "instrument": false, "naive_pdl": true, "event_time_kind": 2},
 {"slack": 3552, "lookahead": 6, "max_active": 8, "event_time_kind": 2}]'
V=$(echo "$V" | python -c "import json,sys; v=json.load(sys.stdin); [x.update(launch_threads=0, dispatcher_cpus=[2]) for x in v]; print(json.dumps(v))")
NREQ=1500 timeout 900 python tools/load_exp.py c3_dispersion 400 "$V" > gpurun_out/ev_light_r2s.jsonl 2> gpurun_out/ev_light_r2s.err; echo "light rc=$?"
NREQ=3000 timeout 900 python tools/load_exp.py c3_dispersion 3000 "$V" > gpurun_out/ev_load_r2s.jsonl 2> gpurun_out/ev_load_r2s.err; echo "load rc=$?"
for f in gpurun_out/ev_light_r2s.jsonl gpurun_out/ev_load_r2s.jsonl; do echo $f; cut -c1-600 $f; done
