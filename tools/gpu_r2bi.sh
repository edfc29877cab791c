#!/bin/bash
# Bench line (C-3) for the autotuner's split gain, M = 64 off; alternating twice.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
for i in 1 2; do
  for gain in 95 80 65; do
    PAELLA_NO_M64=1 PAELLA_SPLIT_GAIN=$gain timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/bench_gain${gain}_$i.json 2> /dev/null
    python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); print(sys.argv[2], d['value'], d['jct_mean_us'], d['jct_p99_us'], d['vs_naive'], d['vs_naive_pdl'], d['x_sat_req_s'], d['req_s_at_slo'], d['e2e']['value'], d['clocks']['sm_mhz'])" gpurun_out/bench_gain${gain}_$i.json $gain
  done
done
