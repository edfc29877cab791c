#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
timeout 900 python -m pytest tests/test_gpu.py -x -q -k "split" > gpurun_out/pytest_r2x.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_r2x.log
for v in both:X dsmem:PAELLA_SPLIT_DSMEM l2:PAELLA_SPLIT_L2; do
  n=${v%%:*}; e=${v#*:}
  env $e=1 PAELLA_AUTOTUNE_LOG=1 timeout 900 python tools/kernel_times.py resnet50 densenet121 inception_v3 mobilenet_v2 > gpurun_out/kt_$n.txt 2> gpurun_out/kt_$n.err; echo "kt $n rc=$?"
  grep "kernels, sum" gpurun_out/kt_$n.txt
  cp gpurun_out/kernel_times.json gpurun_out/kernel_times_$n.json
done
grep -c dsmem gpurun_out/kt_both.err
