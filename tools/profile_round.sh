#!/bin/bash
# Profiling pass of a round (run under gpurun).  ncu serialises launches, so the
# persistent notification mirror warp and the isolated-run gate are disabled
# (PAELLA_NO_PROXY / PAELLA_NO_GATE) for the launch list.  Numbers printed under ncu
# are never bench values.  Split-K choices are autotuned once without ncu and cached
# (PAELLA_SPLITS_FILE) so the profiled runs use the served configuration.
set -x
R=${1:-r1}
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
export PAELLA_SPLITS_FILE=/tmp/paella_splits_$$.txt
rm -f $PAELLA_SPLITS_FILE
timeout 600 python tools/ncu_capture.py c2_mix > /dev/null 2>&1
cp $PAELLA_SPLITS_FILE gpurun_out/splits_${R}.txt
# 1. launch list of a short bench run (every kernel, serialised)
PAELLA_NO_PROXY=1 PAELLA_NO_GATE=1 timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none -c 100000 --csv \
  --log-file /tmp/launches_${R}.csv \
  python bench.py --steps 1 --warmup 3 --reqs 200 --sat-reqs 200 --no-baselines --slo-rhos "" > gpurun_out/bench_under_ncu_${R}.json 2>&1
python tools/ncu_summary.py /tmp/launches_${R}.csv > gpurun_out/launches_${R}_summary.txt 2>&1
gzip -c /tmp/launches_${R}.csv > gpurun_out/launches_${R}.csv.gz
# 2. full sections of every kernel of one request of each C-2 model (served config)
timeout 1500 ncu --set full --import-source on --clock-control none --profile-from-start off \
  -o /tmp/full_${R} python tools/ncu_capture.py c2_mix > gpurun_out/ncu_full_${R}.log 2>&1
ncu -i /tmp/full_${R}.ncu-rep --page raw --csv --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,launch__grid_size,launch__registers_per_thread,sm__throughput.avg.pct_of_peak_sustained_elapsed,lts__t_sector_hit_rate.pct,sm__pipe_tensor_op_hmma_cycles_active.avg.pct_of_peak_sustained_active,gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed > gpurun_out/full_${R}_metrics.csv 2>&1
ls -la /tmp/full_${R}.ncu-rep
