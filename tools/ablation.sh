python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for cfg in c2_mix c3_dispersion; do for pol in sjf rr; do
  timeout 900 python bench.py --config $cfg --policy $pol --slo-rhos "" > gpurun_out/abl_${cfg}_${pol}.json 2>/dev/null; echo "$cfg $pol rc=$?"
done; done
