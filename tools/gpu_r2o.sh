#!/bin/bash
# Diagnosis: Paella vs naive+PDL JCT by launch-ahead depth, light load and ~0.75 load.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
V='[{"naive": true, "instrument": false, "naive_pdl": true},
 {"slack": 1184, "lookahead": 3, "max_active": 8},
 {"slack": 1184, "lookahead": 4, "max_active": 8},
 {"slack": 1184, "lookahead": 5, "max_active": 8},
 {"slack": 1184, "lookahead": 6, "max_active": 8},
 {"slack": 2368, "lookahead": 6, "max_active": 8},
 {"slack": 1184, "lookahead": 6, "max_active": 12}]'
V=$(echo "$V" | python -c "import json,sys; v=json.load(sys.stdin); [x.update(launch_threads=4, dispatcher_cpus=[2]) for x in v]; print(json.dumps(v))")
NREQ=1500 timeout 900 python tools/load_exp.py c3_dispersion 400 "$V" > gpurun_out/la_light_r2o.jsonl 2> gpurun_out/la_light_r2o.err; echo "light rc=$?"
NREQ=4000 timeout 900 python tools/load_exp.py c3_dispersion 4000 "$V" > gpurun_out/la_load_r2o.jsonl 2> gpurun_out/la_load_r2o.err; echo "load rc=$?"
NREQ=4000 timeout 900 python tools/load_exp.py c3_dispersion 5500 "$V" > gpurun_out/la_high_r2o.jsonl 2> gpurun_out/la_high_r2o.err; echo "high rc=$?"
python - <<'PY'
import json
for f in ["gpurun_out/la_light_r2o.jsonl", "gpurun_out/la_load_r2o.jsonl", "gpurun_out/la_high_r2o.jsonl"]:
    print(f)
    for l in open(f):
        d = json.loads(l); v = d["variant"]
        print({k: v[k] for k in v if k not in ("launch_threads", "dispatcher_cpus")}, d["rate"], d["mean_us"], d["p99_us"], d["per_model_mean_us"], d["stop"], d["avg_Q"])
PY
