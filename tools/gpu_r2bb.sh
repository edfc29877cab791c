#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
export PAELLA_SPLITS_FILE=/tmp/splits_dn.txt
timeout 600 python tools/ncu_one_layer.py densenet121 > /dev/null 2>&1   # autotune once, unprofiled
grep "densenet121 4 " /tmp/splits_dn.txt
timeout 900 ncu --profile-from-start off -k regex:k_conv_tc --launch-skip 2 --launch-count 1 --set full --import-source on --clock-control none -o /tmp/dn4 python tools/ncu_one_layer.py densenet121 > gpurun_out/ncu_dn4.log 2>&1; echo "ncu rc=$?"; tail -3 gpurun_out/ncu_dn4.log
ncu -i /tmp/dn4.ncu-rep --page details --csv > gpurun_out/ncu_dn4_details.csv 2>&1
ncu -i /tmp/dn4.ncu-rep --page source --csv --print-source sass > gpurun_out/ncu_dn4_source.csv 2>&1
ncu -i /tmp/dn4.ncu-rep --page raw --csv > gpurun_out/ncu_dn4_raw.csv 2>&1
ls -la gpurun_out/ncu_dn4*
