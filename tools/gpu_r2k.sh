#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
( time timeout 1500 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_r2k.json 2> gpurun_out/bench_r2k.err ) 2> gpurun_out/bench_r2k.time; echo "bench rc=$?"; cat gpurun_out/bench_r2k.json; cat gpurun_out/bench_r2k.time
cp gpurun_out/bench_detail_c3_dispersion_n1.json gpurun_out/bench_detail_c3_r2k.json
timeout 1200 python bench.py --config c2_mix --steps 10 --warmup 3 > gpurun_out/bench_c2_r2k.json 2> gpurun_out/bench_c2_r2k.err; echo "bench c2 rc=$?"; head -c 600 gpurun_out/bench_c2_r2k.json
timeout 1200 python bench.py --arms paella,paella_fifo,paella_ss,paella_ms_kbk,naive,naive_pdl --no-slo --no-c5 --steps 5 --warmup 2 > gpurun_out/bench_table3_r2k.json 2> gpurun_out/bench_table3_r2k.err; echo "table3 rc=$?"
cp gpurun_out/bench_detail_c3_dispersion_n1.json gpurun_out/bench_detail_table3_r2k.json
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref_r2k.json 2> gpurun_out/bench_ref_r2k.err; echo "ref rc=$?"; head -c 400 gpurun_out/bench_ref_r2k.json
du -sh gpurun_out
