#!/bin/bash
# Confirmation of the committed tree: smoke and one bench line.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_confirm.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/smoke_confirm.log
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/bench_confirm.json 2> gpurun_out/bench_confirm.err; echo "bench rc=$?"; head -c 600 gpurun_out/bench_confirm.json
