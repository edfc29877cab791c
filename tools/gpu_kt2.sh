python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "forced_split or isolated_bf16" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
timeout 900 python tools/kernel_times.py resnet18 resnet50 densenet121 > gpurun_out/kt_fence.txt 2>&1
PAELLA_XNOFENCE=1 timeout 900 python tools/kernel_times.py resnet18 resnet50 densenet121 > gpurun_out/kt_nofence.txt 2>&1
