#!/bin/bash
# 128-pixel tiles (KIND_CONV_TC128) for saturating shapes: parity, then TFLOP/s vs 64-pixel tiles.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
timeout 900 python -m pytest tests/test_gpu.py -x -q -k "wide or parity_bf16 or split" > gpurun_out/pytest_r2au.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_r2au.log
timeout 600 python tools/conv_saturating.py > gpurun_out/sat_wide.json 2> gpurun_out/sat_wide.err; echo "sat rc=$?"; cat gpurun_out/sat_wide.json; tail -3 gpurun_out/sat_wide.err
PAELLA_NO_WIDE=1 timeout 600 python tools/conv_saturating.py > gpurun_out/sat_n64.json 2>/dev/null; echo "sat64 rc=$?"; cat gpurun_out/sat_n64.json
