#!/bin/bash
# Diagnosis: host launch throughput; light-load JCT of Paella vs naive+PDL by launch-ahead depth.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o /tmp/lr tools/launch_rate.cu -lcuda -lpthread && timeout 300 /tmp/lr 40000 > gpurun_out/launch_rate_r2n.txt 2>&1; echo "lr rc=$?"; cat gpurun_out/launch_rate_r2n.txt
V='[{"naive": true, "instrument": false, "naive_pdl": true},
 {"slack": 1184, "lookahead": 3, "max_active": 8},
 {"slack": 1184, "lookahead": 6, "max_active": 8},
 {"slack": 1184, "lookahead": 12, "max_active": 8},
 {"slack": 1184, "lookahead": 3, "max_active": 8, "notify": "ring"},
 {"slack": 1184, "lookahead": 3, "max_active": 8, "proxy": false}]'
V=$(echo "$V" | python -c "import json,sys; v=json.load(sys.stdin); [x.update(launch_threads=4, dispatcher_cpus=[2]) for x in v]; print(json.dumps(v))")
NREQ=1500 timeout 900 python tools/load_exp.py c3_dispersion 400 "$V" > gpurun_out/la_light_r2n.jsonl 2> gpurun_out/la_light_r2n.err; echo "light rc=$?"
NREQ=3000 timeout 900 python tools/load_exp.py c3_dispersion 4000 "$V" > gpurun_out/la_load_r2n.jsonl 2> gpurun_out/la_load_r2n.err; echo "load rc=$?"
python - <<'PY'
import json
for f in ["gpurun_out/la_light_r2n.jsonl", "gpurun_out/la_load_r2n.jsonl"]:
    print(f)
    for l in open(f):
        d = json.loads(l); v = d["variant"]
        print({k: v[k] for k in v if k not in ("launch_threads", "dispatcher_cpus")}, d["rate"], d["mean_us"], d["p99_us"], d["per_model_mean_us"], d["stop"], d["avg_Q"])
PY
