#!/bin/bash
# (1) per-SM L2 -> shared-memory fill rate; (2) X_dev / latency / CTAs of the C-3 mix for
# M = 64 on/off x autotuner split gain.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o /tmp/l2bw tools/l2_fill_bw.cu && timeout 300 /tmp/l2bw | tee gpurun_out/l2_fill_bw.txt
for rep in 1 2; do
for m in X PAELLA_NO_M64; do
  for gain in 95 80 65; do
    env $m=1 PAELLA_SPLIT_GAIN=$gain timeout 600 python tools/xdev_ab.py 2>/dev/null | tee -a gpurun_out/xdev_ab.jsonl
  done
done
done
