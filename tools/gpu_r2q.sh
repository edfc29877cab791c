#!/bin/bash
# Timeline of light-load serving (ring mode, G = 1, host decision times).
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
timeout 600 python tools/timeline.py c3_dispersion 300 80 gpurun_out/tl_la6 '{"lookahead": 6, "slack": 3552}' > gpurun_out/tl_la6.json 2> gpurun_out/tl_la6.err; echo "tl rc=$?"; cat gpurun_out/tl_la6.json; tail -3 gpurun_out/tl_la6.err
timeout 600 python tools/timeline.py c3_dispersion 300 80 gpurun_out/tl_la3 '{"lookahead": 3, "slack": 1184}' > gpurun_out/tl_la3.json 2> gpurun_out/tl_la3.err; echo "tl rc=$?"; cat gpurun_out/tl_la3.json
gzip -f gpurun_out/tl_la6.trace.json gpurun_out/tl_la3.trace.json; rm -f gpurun_out/*.evlog
