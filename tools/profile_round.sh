#!/bin/bash
# Profiling pass of a round (run under gpurun).  ncu serialises launches, so the
# persistent notification-proxy warp and the isolated-run gate are disabled
# (PAELLA_NO_PROXY / PAELLA_NO_GATE): the launch list therefore shows the
# direct-write instrumentation variant.  Numbers printed under ncu are never bench
# values.
set -x
R=${1:-r1}
export PAELLA_NO_PROXY=1 PAELLA_NO_GATE=1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 200000 --csv \
  --log-file gpurun_out/launches_${R}.csv \
  python bench.py --steps 1 --warmup 1 --reqs 200 --sat-reqs 200 --no-baselines > gpurun_out/bench_under_ncu_${R}.json 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_conv_tc -s 40 -c 4 \
  -o gpurun_out/conv_full_${R} python tools/gpu_check.py resnet18 > gpurun_out/ncu_full_${R}.log 2>&1
