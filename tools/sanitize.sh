#!/bin/bash
# Sanitizer runs (VERDICT r1 "Sanitizers: no").
#  tsan: the host runtime (dispatcher, launchers, router, channels, policy) built with
#        -fsanitize=thread, driven by the CPU library tests on the fake device -- runs
#        here, no GPU.  Reports go to $OUT/tsan.*; the run fails if any report exists.
#  cuda: compute-sanitizer -- closed on this GPU pool (see below).
set -u
OUT=${OUT:-gpurun_out/sanitize}
mkdir -p "$OUT"
mode=${1:-tsan}
if [ "$mode" = tsan ]; then
  python -m paper_conf_sosp_ngd023_b200.build --tsan > /dev/null || exit 1
  rm -f "$OUT"/tsan.*
  LD_PRELOAD=$(gcc -print-file-name=libtsan.so) \
  TSAN_OPTIONS="halt_on_error=0 report_signal_unsafe=0 suppressions=$PWD/tools/tsan.supp log_path=$PWD/$OUT/tsan" \
  PAELLA_LIB=$PWD/paper_conf_sosp_ngd023_b200/libpaella_tsan.so \
    timeout 1800 python -m pytest tests/test_lib_cpu.py tests/test_router_cpu.py tests/test_faults_cpu.py tests/test_client_process_cpu.py -q -p no:cacheprovider 2>&1 | tail -2
  n=$(cat "$OUT"/tsan.* 2>/dev/null | grep -c "WARNING: ThreadSanitizer")
  echo "tsan reports: $n"
  [ "$n" = 0 ]
else
  # compute-sanitizer is closed on this GPU pool (gpurun answers rc 86: runs under it have
  # left GPUs needing a reset); kernel memory safety is covered by the bounds asserts and
  # the element-by-element parity tests instead (tests/test_gpu.py)
  echo "compute-sanitizer unavailable on this pool"; exit 2
fi
