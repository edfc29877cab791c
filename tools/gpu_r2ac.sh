#!/bin/bash
# A/B on one box: 4-stage ring for every layer (PAELLA_STAGES4) vs deeper rings for narrow layers.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
timeout 600 python -m pytest tests/test_gpu.py -x -q -k "parity_bf16 or split" > gpurun_out/pytest_r2ac.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/pytest_r2ac.log
for r in 1 2; do
for v in st4:PAELLA_STAGES4 deep:X; do
  n=${v%%:*}; e=${v#*:}
  env $e=1 timeout 900 python tools/kernel_times.py resnet50 densenet121 inception_v3 mobilenet_v2 > gpurun_out/kt_${n}_$r.txt 2>/dev/null; echo "kt $n $r rc=$?"
  grep "kernels, sum" gpurun_out/kt_${n}_$r.txt
done
done
