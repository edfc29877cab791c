#!/bin/bash
# Bench line: SRPT-ordered job cap (default) vs arrival-ordered (--cap-fifo), same box.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
timeout 1500 python bench.py --steps 5 --warmup 3 > gpurun_out/bench_capdef.json 2>/dev/null; echo "def rc=$?"; head -c 600 gpurun_out/bench_capdef.json; echo
timeout 1500 python bench.py --steps 5 --warmup 3 --cap-fifo > gpurun_out/bench_capfifo.json 2>/dev/null; echo "fifo rc=$?"; head -c 600 gpurun_out/bench_capfifo.json; echo
