#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
timeout 900 python -m pytest tests/test_gpu.py -x -q -k "split or parity_bf16" > gpurun_out/pytest_r2w.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_r2w.log
rm -f /tmp/sp.txt
PAELLA_SPLIT_DSMEM=1 PAELLA_SPLITS_FILE=/tmp/sp.txt timeout 600 python tools/trace_all_convs.py resnet50 densenet121 > gpurun_out/twA.jsonl 2> gpurun_out/twA.txt
PAELLA_SPLITS_FILE=/tmp/sp.txt timeout 600 python tools/trace_all_convs.py resnet50 densenet121 > gpurun_out/twB.jsonl 2> gpurun_out/twB.txt
PAELLA_SPLIT_NOROT=1 PAELLA_SPLITS_FILE=/tmp/sp.txt timeout 600 python tools/trace_all_convs.py resnet50 densenet121 > gpurun_out/twC.jsonl 2> gpurun_out/twC.txt
PAELLA_SPLIT_RELBAR=1 PAELLA_SPLITS_FILE=/tmp/sp.txt timeout 600 python tools/trace_all_convs.py resnet50 densenet121 > gpurun_out/twD.jsonl 2> gpurun_out/twD.txt
for x in A B C D; do python tools/trace_summary.py gpurun_out/tw$x.txt gpurun_out/tw$x.jsonl > gpurun_out/tw${x}_summary.txt; echo "== $x"; tail -2 gpurun_out/tw${x}_summary.txt; done
