#!/bin/bash
# Dispatcher placement experiment (dedicated core, SCHED_FIFO): C-2 bench
# unpinned, pinned to core 2 (other threads excluded from it), pinned + SCHED_FIFO 50.
set -u
mkdir -p gpurun_out
nproc > gpurun_out/pin_nproc.txt
lscpu | grep -E "NUMA|Model name|^CPU\(s\)" >> gpurun_out/pin_nproc.txt
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/pin_build.log 2>&1
for v in "excl2:--dispatcher-cpu 2:" "excl2fifo:--dispatcher-cpu 2 --dispatcher-fifo 50:" "unpinned2::"; do
  name=${v%%:*}; rest=${v#*:}; flags=${rest%%:*}
  timeout 600 python bench.py $flags > gpurun_out/pin_$name.json 2> gpurun_out/pin_$name.err
  echo "$name rc=$?"
done
