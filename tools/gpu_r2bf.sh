#!/bin/bash
# mbarrier spin (test_wait) vs try_wait in the conv k-block loop: parity under spin, A/B
# phase traces and per-model device time; then the full validation of the default build.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
PAELLA_MBAR_SPIN=1 timeout 900 python -m pytest tests/test_gpu.py -x -q -k "parity or split or wide" > gpurun_out/pytest_spin.log 2>&1; echo "pytest spin rc=$?"; tail -2 gpurun_out/pytest_spin.log
rm -f /tmp/sp.txt
PAELLA_SPLITS_FILE=/tmp/sp.txt timeout 600 python tools/trace_all_convs.py resnet50 densenet121 > gpurun_out/spinA.jsonl 2> gpurun_out/spinA.txt
PAELLA_MBAR_SPIN=1 PAELLA_SPLITS_FILE=/tmp/sp.txt timeout 600 python tools/trace_all_convs.py resnet50 densenet121 > gpurun_out/spinB.jsonl 2> gpurun_out/spinB.txt
for x in A B; do python tools/trace_summary.py gpurun_out/spin$x.txt gpurun_out/spin$x.jsonl > gpurun_out/spin${x}_summary.txt; echo "== $x"; tail -3 gpurun_out/spin${x}_summary.txt; grep "^densenet121 *4 \|^resnet50 *5 " gpurun_out/spin${x}_summary.txt; done
for v in X PAELLA_MBAR_SPIN X PAELLA_MBAR_SPIN; do env $v=1 timeout 600 python tools/kernel_times.py resnet50 densenet121 inception_v3 mobilenet_v2 2>/dev/null | grep "kernels, sum"; done
bash tools/gpu_r2final.sh
