#!/bin/bash
# ncu --set full of the SpMV and Gram kernels of one C2 solve (+ the launch list of a bench run)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 ncu --set full --clock-control none --import-source on -k regex:spmv_sell32 -s 60 -c 1 -o gpurun_out/prof_spmv python tools/kprof.py > gpurun_out/prof_spmv.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:gram -s 6 -c 1 -o gpurun_out/prof_gram python tools/kprof.py > gpurun_out/prof_gram.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:rows_pipe -s 20 -c 2 -o gpurun_out/prof_rows python tools/kprof.py > gpurun_out/prof_rows.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:xty_pipe -s 6 -c 2 -o gpurun_out/prof_xty python tools/kprof.py > gpurun_out/prof_xty.log 2>&1
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu > gpurun_out/bench.log 2>&1
