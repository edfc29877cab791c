#!/bin/bash
# Experiment: 8-stage ring at one CTA/SM for the convs with >= 8 k-blocks (PAELLA_DEEP_RING).
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
rm -f /tmp/sp.txt
PAELLA_SPLITS_FILE=/tmp/sp.txt timeout 600 python tools/trace_all_convs.py resnet50 densenet121 > gpurun_out/dpA.jsonl 2> gpurun_out/dpA.txt
PAELLA_DEEP_RING=1 PAELLA_SPLITS_FILE=/tmp/sp.txt timeout 600 python tools/trace_all_convs.py resnet50 densenet121 > gpurun_out/dpB.jsonl 2> gpurun_out/dpB.txt
for x in A B; do python tools/trace_summary.py gpurun_out/dp$x.txt gpurun_out/dp$x.jsonl > gpurun_out/dp${x}_summary.txt; echo "== $x"; tail -2 gpurun_out/dp${x}_summary.txt; grep "^densenet121 *4 \|^resnet50 *5 \|^resnet50 *50 " gpurun_out/dp${x}_summary.txt; done
PAELLA_DEEP_RING=1 timeout 600 python -m pytest tests/test_gpu.py -x -q -k "split" 2>&1 | tail -1
for v in X PAELLA_DEEP_RING; do env $v=1 timeout 600 python tools/kernel_times.py resnet50 densenet121 inception_v3 mobilenet_v2 2>/dev/null | grep "kernels, sum"; done
