#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
timeout 2400 python tools/rho_sweep.py r2ap > gpurun_out/rho_sweep_r2ap.log 2>&1; echo "rho rc=$?"
python tools/rho_summary.py gpurun_out/rho_sweep_r2ap.jsonl > gpurun_out/rho_sweep_r2ap.md; cat gpurun_out/rho_sweep_r2ap.md
