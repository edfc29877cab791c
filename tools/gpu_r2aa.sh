#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
( time timeout 1500 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_r2aa.json 2> gpurun_out/bench_r2aa.err ) 2> gpurun_out/bench_r2aa.time; echo "bench rc=$?"; head -c 1500 gpurun_out/bench_r2aa.json; cat gpurun_out/bench_r2aa.time
cp gpurun_out/bench_detail_c3_dispersion_n1.json gpurun_out/bench_detail_c3_r2aa.json
timeout 1200 python bench.py --config c2_mix --steps 10 --warmup 3 > gpurun_out/bench_c2_r2aa.json 2> gpurun_out/bench_c2_r2aa.err; echo "bench c2 rc=$?"; head -c 900 gpurun_out/bench_c2_r2aa.json
cp gpurun_out/bench_detail_c2_mix_n1.json gpurun_out/bench_detail_c2_r2aa.json
