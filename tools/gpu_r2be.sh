#!/bin/bash
# UMMA M = 64 for narrow layers: parity, then A/B (PAELLA_NO_M64) phase traces and per-model time.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
timeout 1200 python -m pytest tests/test_gpu.py -x -q -k "parity or split or wide" > gpurun_out/pytest_r2be.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_r2be.log
rm -f /tmp/sp.txt
PAELLA_NO_M64=1 PAELLA_SPLITS_FILE=/tmp/sp.txt timeout 600 python tools/trace_all_convs.py resnet50 densenet121 mobilenet_v2 > gpurun_out/m64A.jsonl 2> gpurun_out/m64A.txt
PAELLA_SPLITS_FILE=/tmp/sp.txt timeout 600 python tools/trace_all_convs.py resnet50 densenet121 mobilenet_v2 > gpurun_out/m64B.jsonl 2> gpurun_out/m64B.txt
for x in A B; do python tools/trace_summary.py gpurun_out/m64$x.txt gpurun_out/m64$x.jsonl > gpurun_out/m64${x}_summary.txt; echo "== $x"; tail -3 gpurun_out/m64${x}_summary.txt; grep "^densenet121 *4 \|^resnet50 *5 " gpurun_out/m64${x}_summary.txt; done
for v in PAELLA_NO_M64 X; do env $v=1 timeout 600 python tools/kernel_times.py resnet50 densenet121 inception_v3 mobilenet_v2 2>/dev/null | grep "kernels, sum"; done
