#!/bin/bash
# Sanitizer runs (VERDICT r1 "Sanitizers: no").
#  tsan: the host runtime (dispatcher, launchers, router, channels, policy) built with
#        -fsanitize=thread, driven by the CPU library tests on the fake device -- runs
#        here, no GPU.  Reports go to $OUT/tsan.*; the run fails if any report exists.
#  cuda: compute-sanitizer memcheck / racecheck / synccheck on the isolated parity tests
#        and smoke (GPU box only).
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
  for tool in memcheck racecheck synccheck; do
    sel="isolated_bf16_parity and (toy or resnet18 or mobilenet_v2 or densenet121)"
    [ $tool = memcheck ] && sel="isolated or wide_tile or forced_split_k"
    timeout 1500 compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 20 \
      python -m pytest tests/test_gpu.py -x -q -k "$sel" -p no:cacheprovider \
      > "$OUT/cs_$tool.log" 2>&1
    echo "$tool tests rc=$?"; tail -3 "$OUT/cs_$tool.log"
  done
  timeout 900 compute-sanitizer --tool memcheck --error-exitcode 9 python -c "import __graft_entry__ as g; g.smoke()" \
    > "$OUT/cs_smoke.log" 2>&1; echo "memcheck smoke rc=$?"; tail -3 "$OUT/cs_smoke.log"
fi
