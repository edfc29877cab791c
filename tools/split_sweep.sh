python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
for cfg in "12 4" "6 2" "4 2" "8 3"; do set -- $cfg; PAELLA_SPLIT_MIN_NK=$1 PAELLA_SPLIT_MIN_STAGES=$2 timeout 300 python tools/kernel_times.py > gpurun_out/kt_split_$1_$2.txt 2>&1; done
