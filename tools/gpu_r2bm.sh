#!/bin/bash
# Bench line (C-3) for split gain 65 (default) vs 50 vs no split-K at all; alternating twice.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
for i in 1 2; do
  for v in PAELLA_SPLIT_GAIN=65 PAELLA_SPLIT_GAIN=50 PAELLA_NOSPLIT=1; do
    f=gpurun_out/bench_${v%%=*}_${v##*=}_$i.json
    env $v timeout 900 python bench.py --steps 5 --warmup 3 > $f 2> /dev/null
    python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); print(sys.argv[2], d['value'], d['jct_mean_us'], d['jct_p99_us'], d['vs_naive'], d['vs_naive_pdl'], d['x_sat_req_s'], d['req_s_at_slo'], d['e2e']['value'])" $f $v
  done
done
