python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
for cfg in c3_dispersion c2_mix; do
  timeout 900 python bench.py --config $cfg --online-tbar --slo-rhos "" > gpurun_out/online_${cfg}.json 2>/dev/null; echo "$cfg rc=$?"
done
