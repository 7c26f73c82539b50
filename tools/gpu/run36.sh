#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 ncu --set full --clock-control none --import-source on -k regex:"spmv_dia" -s 400 -c 1 -o gpurun_out/prof_spmv16 python tools/kprof.py --opt spmv=16 > gpurun_out/prof_spmv16.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:"trsm_ring" -s 20 -c 1 -o gpurun_out/prof_trsm python tools/kprof.py > /dev/null 2>&1
timeout 600 python bench.py --config C3 --steps 3 --warmup 3 --no-cpu > gpurun_out/bench36_C3.log 2>&1
timeout 300 python bench.py --config C1 --steps 5 --warmup 3 --no-cpu > gpurun_out/bench36_C1.log 2>&1
