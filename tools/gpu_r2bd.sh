#!/bin/bash
# Timing experiment: is the MMA thread's per-stage proxy fence the loop bottleneck?
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
rm -f /tmp/sp.txt
PAELLA_SPLITS_FILE=/tmp/sp.txt timeout 600 python tools/trace_all_convs.py resnet50 densenet121 > gpurun_out/pfA.jsonl 2> gpurun_out/pfA.txt
PAELLA_NO_PROXY_FENCE=1 PAELLA_SPLITS_FILE=/tmp/sp.txt timeout 600 python tools/trace_all_convs.py resnet50 densenet121 > gpurun_out/pfB.jsonl 2> gpurun_out/pfB.txt
for x in A B; do python tools/trace_summary.py gpurun_out/pf$x.txt gpurun_out/pf$x.jsonl > gpurun_out/pf${x}_summary.txt; echo "== $x"; tail -2 gpurun_out/pf${x}_summary.txt; grep "^densenet121 *4 \|^resnet50 *5 \|^resnet50 *50 " gpurun_out/pf${x}_summary.txt; done
