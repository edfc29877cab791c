#!/bin/bash
# Same-box A/B of the bench line with and without the M = 64 conv (alternating), then the
# compute-sanitizer runs.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
for i in 1 2; do
  for v in X PAELLA_NO_M64; do
    env $v=1 timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/bench_ab_${v}_$i.json 2> /dev/null
    python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); print(sys.argv[2], d['value'], d['jct_mean_us'], d['jct_p99_us'], d['x_sat_req_s'], d['req_s_at_slo'], d['clocks']['sm_mhz'])" gpurun_out/bench_ab_${v}_$i.json $v
  done
done
OUT=gpurun_out/sanitize bash tools/sanitize.sh cuda
