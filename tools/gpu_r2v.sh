#!/bin/bash
# split-K in L2 (bulk f32 reductions) vs DSMEM: parity, then phase traces with identical splits.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
timeout 900 python -m pytest tests/test_gpu.py -x -q -k "parity or split" > gpurun_out/pytest_r2v.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_r2v.log
rm -f /tmp/sp.txt
PAELLA_SPLIT_DSMEM=1 PAELLA_SPLITS_FILE=/tmp/sp.txt timeout 600 python tools/trace_all_convs.py resnet50 densenet121 > gpurun_out/tcA.jsonl 2> gpurun_out/tcA.txt; echo "A rc=$?"
PAELLA_SPLITS_FILE=/tmp/sp.txt timeout 600 python tools/trace_all_convs.py resnet50 densenet121 > gpurun_out/tcB.jsonl 2> gpurun_out/tcB.txt; echo "B rc=$?"
PAELLA_AUTOTUNE_LOG=1 timeout 600 python tools/trace_all_convs.py resnet50 densenet121 > gpurun_out/tcC.jsonl 2> gpurun_out/tcC.txt; echo "C rc=$?"
cp /tmp/sp.txt gpurun_out/splits_dsmem.txt
for x in A B C; do python tools/trace_summary.py gpurun_out/tc$x.txt gpurun_out/tc$x.jsonl > gpurun_out/tc${x}_summary.txt; echo "== $x"; tail -2 gpurun_out/tc${x}_summary.txt; done
