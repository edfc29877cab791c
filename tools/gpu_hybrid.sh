python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1


timeout 300 python tools/hybrid_exp.py 500 2000 6000 > gpurun_out/hybrid_r1b.jsonl 2> gpurun_out/hybrid.err
