python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for th in 20 5 1; do timeout 900 python bench.py --config c3_dispersion --theta $th --slo-rhos "" > gpurun_out/bench_c3_theta$th.json 2>/dev/null; done
