#!/bin/bash
# Deeper stage rings for narrow layers: parity, per-layer phases, per-model device time.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_r2ab.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu_r2ab.log
PAELLA_AUTOTUNE_LOG=1 timeout 900 python tools/trace_all_convs.py resnet50 densenet121 mobilenet_v2 > gpurun_out/tsE.jsonl 2> gpurun_out/tsE.txt; echo "trace rc=$?"
python tools/trace_summary.py gpurun_out/tsE.txt gpurun_out/tsE.jsonl > gpurun_out/tsE_summary.txt; tail -3 gpurun_out/tsE_summary.txt
PAELLA_AUTOTUNE_LOG=1 timeout 900 python tools/kernel_times.py resnet50 densenet121 inception_v3 mobilenet_v2 > gpurun_out/kt_stages.txt 2> gpurun_out/kt_stages.err; echo "kt rc=$?"
grep "kernels, sum\|slowdown" gpurun_out/kt_stages.txt
