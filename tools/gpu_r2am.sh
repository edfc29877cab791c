#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
timeout 600 python tools/timeline.py c1_toy 300 100 /tmp/tlt > gpurun_out/tlt.json 2> gpurun_out/tlt.err; echo "toy rc=$?"
python -c "
import sys; sys.path.insert(0, 'tools'); import timeline
timeline.dump_jobs('/tmp/tlt.evlog', ['toy'], 6)"
timeout 600 python tools/timeline.py c3_dispersion 300 40 /tmp/tlc > gpurun_out/tlc.json 2> gpurun_out/tlc.err; echo "c3 rc=$?"
python -c "
import sys; sys.path.insert(0, 'tools'); import timeline
timeline.dump_jobs('/tmp/tlc.evlog', ['resnet50', 'densenet121', 'inception_v3', 'mobilenet_v2'], 3)" | head -150
