#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
timeout 900 python tools/trace_all_convs.py resnet50 mobilenet_v2 densenet121 inception_v3 > gpurun_out/tc_layers.jsonl 2> gpurun_out/tc_trace.txt; echo "trace rc=$?"
python tools/trace_summary.py gpurun_out/tc_trace.txt gpurun_out/tc_layers.jsonl > gpurun_out/tc_summary.txt; tail -5 gpurun_out/tc_summary.txt
