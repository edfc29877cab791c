#!/bin/bash
# Independent accumulation chains: k-block it accumulates into TMEM accumulator it % A
# (A = 1 default, 2, 4; build variants libpaella_acc{2,4}.so), summed in the epilogue.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
D=$PWD/paper_conf_sosp_ngd023_b200
for v in acc2 acc4; do
  PAELLA_LIB=$D/libpaella_$v.so timeout 900 python -m pytest tests/test_gpu.py -x -q -k "isolated_bf16 or split" > gpurun_out/pytest_$v.log 2>&1; echo "pytest $v rc=$?"; tail -1 gpurun_out/pytest_$v.log
done
rm -f /tmp/sp.txt
for v in paella paella_acc2 paella_acc4; do
  PAELLA_LIB=$D/lib$v.so PAELLA_SPLITS_FILE=/tmp/sp.txt timeout 600 python tools/trace_all_convs.py resnet50 inception_v3 > gpurun_out/acc_$v.jsonl 2> gpurun_out/acc_$v.txt
  python tools/trace_summary.py gpurun_out/acc_$v.txt gpurun_out/acc_$v.jsonl > gpurun_out/acc_${v}_summary.txt; echo "== $v"; tail -2 gpurun_out/acc_${v}_summary.txt
done
for v in paella paella_acc2 paella_acc4; do PAELLA_LIB=$D/lib$v.so PAELLA_SPLITS_FILE=/tmp/sp.txt timeout 600 python tools/kernel_times.py resnet50 densenet121 inception_v3 mobilenet_v2 2>/dev/null | grep "kernels, sum"; done
for v in paella paella_acc2 paella_acc4; do PAELLA_LIB=$D/lib$v.so timeout 600 python tools/xdev_ab.py 2>/dev/null; done
