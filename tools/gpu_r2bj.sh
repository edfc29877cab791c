#!/bin/bash
# Activations by TMA im2col (LF_TMA_B): parity, then A/B (PAELLA_NO_TMA_B) phase traces and
# per-model device time with the same split factors.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
timeout 900 python -m pytest tests/test_gpu.py -x -q -k "parity or split or wide or c1_toy" > gpurun_out/pytest_tmab.log 2>&1; echo "pytest rc=$?"; tail -15 gpurun_out/pytest_tmab.log | grep -v "^$" | tail -8
rm -f /tmp/sp.txt
PAELLA_NO_TMA_B=1 PAELLA_SPLITS_FILE=/tmp/sp.txt timeout 600 python tools/trace_all_convs.py resnet50 inception_v3 > gpurun_out/tmabA.jsonl 2> gpurun_out/tmabA.txt
PAELLA_SPLITS_FILE=/tmp/sp.txt timeout 600 python tools/trace_all_convs.py resnet50 inception_v3 > gpurun_out/tmabB.jsonl 2> gpurun_out/tmabB.txt
for x in A B; do python tools/trace_summary.py gpurun_out/tmab$x.txt gpurun_out/tmab$x.jsonl > gpurun_out/tmab${x}_summary.txt; echo "== $x"; tail -3 gpurun_out/tmab${x}_summary.txt; grep "^resnet50 *5 \|^inception_v3 *[0-9]* " gpurun_out/tmab${x}_summary.txt | head -4; done
for v in PAELLA_NO_TMA_B X; do env $v=1 PAELLA_SPLITS_FILE=/tmp/sp.txt timeout 600 python tools/kernel_times.py resnet50 densenet121 inception_v3 mobilenet_v2 2>/dev/null | grep "kernels, sum\|conv_tcgen"; done
for v in PAELLA_NO_TMA_B X; do env $v=1 timeout 600 python tools/xdev_ab.py 2>/dev/null; done
