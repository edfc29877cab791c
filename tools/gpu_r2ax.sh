#!/bin/bash
# 256-pixel tiles, one CTA per SM (PAELLA_WIDE=256) vs 128-pixel tiles at saturating shapes.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
PAELLA_WIDE=256 timeout 600 python -m pytest tests/test_gpu.py -x -q -k "wide" > gpurun_out/pytest_r2ax.log 2>&1; echo "pytest256 rc=$?"; tail -2 gpurun_out/pytest_r2ax.log
timeout 600 python -m pytest tests/test_gpu.py -x -q -k "wide" 2>&1 | tail -1
PAELLA_WIDE=256 timeout 600 python tools/conv_saturating.py > gpurun_out/sat_n256.json 2> gpurun_out/sat_n256.err; echo "sat256 rc=$?"; cat gpurun_out/sat_n256.json; tail -2 gpurun_out/sat_n256.err
timeout 600 python tools/conv_saturating.py > gpurun_out/sat_n128b.json 2>/dev/null; echo "sat128 rc=$?"; cat gpurun_out/sat_n128b.json
