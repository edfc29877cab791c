# one build -> parity -> per-kernel times -> short bench iteration (under gpurun)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -s > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
PAELLA_AUTOTUNE_LOG=1 timeout 900 python tools/kernel_times.py > gpurun_out/kernel_times.txt 2> gpurun_out/autotune.log
timeout 900 python bench.py ${BENCH_ARGS} > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
