#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_r2av.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu_r2av.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r2av.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/smoke_r2av.log
( time timeout 1500 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_r2av.json 2> gpurun_out/bench_r2av.err ) 2> gpurun_out/bench_r2av.time; echo "bench rc=$?"; head -c 1500 gpurun_out/bench_r2av.json; cat gpurun_out/bench_r2av.time
cp gpurun_out/bench_detail_c3_dispersion_n1.json gpurun_out/bench_detail_c3_r2av.json
timeout 1200 python bench.py --config c2_mix --steps 10 --warmup 3 > gpurun_out/bench_c2_r2av.json 2> gpurun_out/bench_c2_r2av.err; echo "bench c2 rc=$?"; head -c 900 gpurun_out/bench_c2_r2av.json
cp gpurun_out/bench_detail_c2_mix_n1.json gpurun_out/bench_detail_c2_r2av.json
