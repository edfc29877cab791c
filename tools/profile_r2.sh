#!/bin/bash
# Round-2 profiling pass (run under gpurun).  The library switches the persistent
# notification warp and the timing gate off by itself under Nsight Compute.  Numbers
# printed under ncu are never bench values.  Reports stay in /tmp; only CSV/text
# summaries go to gpurun_out (the pull-back limit is 64 MiB).
R=${1:-r2}
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
export PAELLA_SPLITS_FILE=/tmp/paella_splits_$$.txt
timeout 600 python tools/ncu_capture.py c3_dispersion > /dev/null 2>&1     # autotune once, unprofiled
cp $PAELLA_SPLITS_FILE gpurun_out/splits_${R}.txt
# 0. the driver's step: smoke() under ncu must finish
( time timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file /tmp/launches_smoke.csv \
    python -c "import __graft_entry__ as g; g.smoke()" ) > gpurun_out/ncu_smoke_${R}.log 2>&1; echo "ncu smoke rc=$?"
tail -4 gpurun_out/ncu_smoke_${R}.log
# 1. launch list of the C-3 mix as served (paella arm, then naive arm), serialised
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv \
  --log-file /tmp/launches_${R}.csv python tools/ncu_serve.py 150 > gpurun_out/ncu_serve_${R}.log 2>&1
echo "ncu serve rc=$?"
python tools/ncu_summary.py /tmp/launches_${R}.csv > gpurun_out/launches_${R}_summary.txt 2>&1
gzip -c /tmp/launches_${R}.csv > gpurun_out/launches_${R}.csv.gz; ls -la gpurun_out/launches_${R}.csv.gz
# 2. full sections of the conv kernels of one request of each C-3 model (served configuration)
timeout 1500 ncu --set full --import-source on --clock-control none --profile-from-start off -k regex:k_conv_tc \
  -o /tmp/full_${R} python tools/ncu_capture.py c3_dispersion > gpurun_out/ncu_full_${R}.log 2>&1
echo "ncu full rc=$?"
ncu -i /tmp/full_${R}.ncu-rep --page raw --csv --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,launch__grid_size,launch__registers_per_thread,sm__throughput.avg.pct_of_peak_sustained_elapsed,lts__t_sector_hit_rate.pct,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed,gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed,gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed > gpurun_out/full_${R}_metrics.csv 2>&1
ls -la gpurun_out | head -40
du -sh gpurun_out
