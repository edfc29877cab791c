#!/bin/bash
# Timeline of light-load serving, ring mode with one record per launch and type (G = 16:
# the record at count == grid = last block placed / last block exited), host decision times.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
for v in la6:'{"lookahead": 6, "slack": 3552, "group": 16}' la3:'{"lookahead": 3, "slack": 1184, "group": 16}' la6c:'{"lookahead": 6, "slack": 3552, "group": 16, "max_active": 0}'; do
  n=${v%%:*}; j=${v#*:}
  timeout 600 python tools/timeline.py c3_dispersion 300 80 gpurun_out/tlg_$n "$j" > gpurun_out/tlg_$n.json 2> gpurun_out/tlg_$n.err; echo "tl $n rc=$?"; cat gpurun_out/tlg_$n.json; tail -2 gpurun_out/tlg_$n.err
done
gzip -f gpurun_out/tlg_*.trace.json; rm -f gpurun_out/*.evlog
