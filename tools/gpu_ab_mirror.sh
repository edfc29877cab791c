#!/bin/bash
# A/B: mirror publishing the summed counter table (new) vs the 4 tables (old), same box.
run() {
  tag=$1
  python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$tag.log 2>&1; echo "build $tag rc=$?"
  V='[{"slack": 3552, "lookahead": 6, "lookahead_unplaced": true, "max_active": 8, "launch_threads": 8, "dispatcher_cpus": [2]}]'
  for lam in 400 4000 6000; do
    n=$([ $lam = 400 ] && echo 1500 || echo 4000)
    NREQ=$n timeout 600 python tools/load_exp.py c3_dispersion $lam "$V" > gpurun_out/ab_${tag}_$lam.jsonl 2>/dev/null
    python -c "
import json
for l in open('gpurun_out/ab_${tag}_$lam.jsonl'):
    d=json.loads(l); print('  $tag $lam', d['mean_us'], d['p99_us'], d['per_model_mean_us'])"
  done
  timeout 300 python tools/timeline.py c1_toy 300 200 /tmp/tl_$tag > gpurun_out/tl_$tag.json 2>/dev/null; cut -c1-400 gpurun_out/tl_$tag.json
}
mkdir -p /tmp/new && cp paper_conf_sosp_ngd023_b200/csrc/kernels_simt.cu paper_conf_sosp_ngd023_b200/csrc/engine.cpp /tmp/new/
timeout 900 python -m pytest tests/test_gpu.py -x -q -k "serving_parity" > gpurun_out/pytest_ab.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/pytest_ab.log
run new
cp ab_old/kernels_simt.cu ab_old/engine.cpp paper_conf_sosp_ngd023_b200/csrc/
run old
cp /tmp/new/kernels_simt.cu /tmp/new/engine.cpp paper_conf_sosp_ngd023_b200/csrc/
run new2
