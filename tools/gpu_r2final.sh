#!/bin/bash
# Final validation: GPU tests, smoke, smoke under ncu (the driver's step), bench lines.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_final.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu_final.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_final.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/smoke_final.log
( time timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file /tmp/launches_smoke.csv python -c "import __graft_entry__ as g; g.smoke()" ) > gpurun_out/ncu_smoke_final.log 2>&1; echo "ncu smoke rc=$?"; tail -4 gpurun_out/ncu_smoke_final.log; grep -c '"k_' /tmp/launches_smoke.csv
( time timeout 1500 python bench.py --steps 5 --warmup 3 > gpurun_out/bench_final.json 2> gpurun_out/bench_final.err ) 2> gpurun_out/bench_final.time; echo "bench rc=$?"; head -c 700 gpurun_out/bench_final.json; cat gpurun_out/bench_final.time
cp gpurun_out/bench_detail_c3_dispersion_n1.json gpurun_out/bench_detail_c3_final.json
