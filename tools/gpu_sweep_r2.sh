#!/bin/bash
# Round-2 load sweeps: CFG (c3_dispersion|c2_mix) at LAM req/s, variants from VAR (json file)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
export PAELLA_SPLITS_FILE=/tmp/paella_splits_sweep.txt
V=$(cat ${VAR:-tools/variants_r2.json})
NREQ=${NREQ:-4000} timeout 2400 python tools/load_exp.py ${CFG:-c3_dispersion} ${LAM:-4800} "$V" > gpurun_out/sweep_${TAG:-r2}.jsonl 2> gpurun_out/sweep_${TAG:-r2}.err
echo "rc=$?"
