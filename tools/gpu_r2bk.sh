#!/bin/bash
# Stage-ring depth with both operands by TMA: 4 stages (96 KB, 2 CTAs/SM) vs 8 (192 KB,
# 1 CTA/SM; libpaella_ring8.so = PAELLA_DEFINES=-DPAELLA_TC_STAGES=8).
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
R8=$PWD/paper_conf_sosp_ngd023_b200/libpaella_ring8.so
PAELLA_LIB=$R8 timeout 900 python -m pytest tests/test_gpu.py -x -q -k "isolated_bf16 or split or wide" > gpurun_out/pytest_ring8.log 2>&1; echo "pytest ring8 rc=$?"; tail -2 gpurun_out/pytest_ring8.log
rm -f /tmp/sp.txt
PAELLA_SPLITS_FILE=/tmp/sp.txt timeout 600 python tools/trace_all_convs.py resnet50 inception_v3 > gpurun_out/r8A.jsonl 2> gpurun_out/r8A.txt
PAELLA_LIB=$R8 PAELLA_SPLITS_FILE=/tmp/sp.txt timeout 600 python tools/trace_all_convs.py resnet50 inception_v3 > gpurun_out/r8B.jsonl 2> gpurun_out/r8B.txt
for x in A B; do python tools/trace_summary.py gpurun_out/r8$x.txt gpurun_out/r8$x.jsonl > gpurun_out/r8${x}_summary.txt; echo "== $x"; tail -2 gpurun_out/r8${x}_summary.txt; done
for v in X PAELLA_LIB=$R8; do env $v PAELLA_SPLITS_FILE=/tmp/sp.txt timeout 600 python tools/kernel_times.py resnet50 densenet121 inception_v3 mobilenet_v2 2>/dev/null | grep "kernels, sum"; done
for v in X PAELLA_LIB=$R8; do env $v timeout 600 python tools/xdev_ab.py 2>/dev/null; done
for v in X PAELLA_LIB=$R8; do
  env $v timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/bench_r8_$(echo $v | cut -c1-6).json 2> /dev/null
  python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); print(sys.argv[2], d['value'], d['jct_mean_us'], d['jct_p99_us'], d['vs_naive'], d['x_sat_req_s'], d['req_s_at_slo'])" gpurun_out/bench_r8_$(echo $v | cut -c1-6).json $v
done
