#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_r2f.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu_r2f.log
timeout 900 python tools/hol_exp.py r2f 300 > gpurun_out/hol_r2f.log 2>&1; echo "hol rc=$?"; tail -2 gpurun_out/hol_r2f.log
timeout 1500 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_r2f.json 2> gpurun_out/bench_r2f.err; echo "bench rc=$?"; cat gpurun_out/bench_r2f.json
timeout 1200 python tools/rho_sweep.py r2f > gpurun_out/rho_sweep_r2f.log 2>&1; echo "rho rc=$?"
du -sh gpurun_out
