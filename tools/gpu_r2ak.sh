#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
timeout 600 python tools/timeline.py c1_toy 300 200 gpurun_out/tlc_toy > gpurun_out/tlc_toy.json 2> gpurun_out/tlc_toy.err; echo "toy rc=$?"; cat gpurun_out/tlc_toy.json; tail -2 gpurun_out/tlc_toy.err
timeout 600 python tools/timeline.py c3_dispersion 300 100 gpurun_out/tlc_c3 > gpurun_out/tlc_c3.json 2> gpurun_out/tlc_c3.err; echo "c3 rc=$?"; cat gpurun_out/tlc_c3.json; tail -2 gpurun_out/tlc_c3.err
rm -f gpurun_out/*.evlog
