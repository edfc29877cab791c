#!/bin/bash
# Bench line with launch-ahead 6 / B = 3552; the GPU tests of the bench configuration.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
timeout 900 python -m pytest tests/test_gpu.py -x -q -k "bench_arm or replay" > gpurun_out/pytest_r2t.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_r2t.log
( time timeout 1500 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_r2t.json 2> gpurun_out/bench_r2t.err ) 2> gpurun_out/bench_r2t.time; echo "bench rc=$?"; head -c 1200 gpurun_out/bench_r2t.json; cat gpurun_out/bench_r2t.time
cp gpurun_out/bench_detail_c3_dispersion_n1.json gpurun_out/bench_detail_c3_r2t.json
