python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 300 python tools/trace_conv.py resnet50 1 4 5 6 13 15 45 47 48 > gpurun_out/trace_r50.log 2>&1
timeout 300 python tools/trace_conv.py resnet18 1 5 > gpurun_out/trace_r18.log 2>&1
timeout 900 python tools/kernel_times.py > gpurun_out/kernel_times_r1b.txt 2>&1
