python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for cfg in c3_dispersion c2_mix; do
  timeout 900 python bench.py --config $cfg --theta 1000000000000000 --slo-rhos "" > gpurun_out/thinf_${cfg}.json 2>/dev/null; echo "$cfg rc=$?"
done
