python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for d in 0 2000 5000 10000 20000 50000; do
  timeout 600 python bench.py --no-baselines --slo-rhos "" --decide-delay-ns $d --steps 3 > gpurun_out/delay_$d.json 2>/dev/null; echo "delay $d rc=$?"
done
