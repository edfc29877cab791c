#!/bin/bash
# Round-2 GPU pass: tests, smoke, profiler env check, bench
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1800 python -m pytest tests -m gpu -x -q ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pytest_gpu_${TAG}.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu_${TAG}.log
timeout 300 python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke_${TAG}.log 2>&1; echo "smoke rc=$?"
timeout 120 ncu --metrics gpu__time_duration.sum --clock-control none -c 5 bash -c "env | grep -i -E 'inject|preload|nsight|nv_' | sed s/^/INJ:/" > gpurun_out/ncu_env_${TAG}.log 2>&1
grep INJ gpurun_out/ncu_env_${TAG}.log
if [ -z "$NOBENCH" ]; then
timeout 1500 python bench.py --steps ${STEPS:-10} --warmup 3 > gpurun_out/bench_${TAG}.json 2> gpurun_out/bench_${TAG}.err; echo "bench rc=$?"
tail -c 3000 gpurun_out/bench_${TAG}.json
fi
if [ -n "$KT" ]; then
timeout 900 python tools/kernel_times.py > gpurun_out/kernel_times_${TAG}.txt 2>&1; echo "kt rc=$?"; tail -2 gpurun_out/kernel_times_${TAG}.txt
cp gpurun_out/kernel_times.json gpurun_out/kernel_times_${TAG}.json
fi
if [ -n "$KTSYS" ]; then
PAELLA_LAST_SYS=1 timeout 900 python tools/kernel_times.py > gpurun_out/kernel_times_${TAG}_sys.txt 2>&1; echo "ktsys rc=$?"; tail -1 gpurun_out/kernel_times_${TAG}_sys.txt
cp gpurun_out/kernel_times.json gpurun_out/kernel_times_${TAG}_sys.json
fi
if [ -n "$SWEEP" ]; then
VAR=$SWEEP TAG=${TAG}_sweep LAM=${LAM:-3600} bash tools/gpu_sweep_r2.sh
fi
if [ -n "$C5" ]; then
timeout 600 python tools/c5_table.py ${TAG} > gpurun_out/c5_${TAG}.txt 2>&1; echo "c5 rc=$?"; tail -3 gpurun_out/c5_${TAG}.txt
fi
