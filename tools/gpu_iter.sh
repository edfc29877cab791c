# one build -> parity -> trace -> per-kernel times -> short bench iteration (under gpurun)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -s > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
timeout 300 python tools/trace_conv.py resnet50 5 45 47 > gpurun_out/trace_r50.log 2>&1
timeout 900 python tools/kernel_times.py > gpurun_out/kernel_times.txt 2>&1
timeout 900 python bench.py ${BENCH_ARGS} > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
