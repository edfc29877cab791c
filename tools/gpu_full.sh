# build -> GPU tests -> per-kernel times -> C-2 and C-3 bench lines (under gpurun)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -s > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
PAELLA_AUTOTUNE_LOG=1 timeout 900 python tools/kernel_times.py > gpurun_out/kernel_times.txt 2> gpurun_out/autotune.log
timeout 900 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err; echo "bench c2 rc=$?"
timeout 1200 python bench.py --config c3_dispersion > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err; echo "bench c3 rc=$?"
