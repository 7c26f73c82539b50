#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 ncu --set full --clock-control none --import-source on -k regex:spmv_ring -s 40 -c 1 -o gpurun_out/prof_ring python tools/kprof.py --opt spmv=10 > gpurun_out/prof_ring.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:spmv_sell32_persist -s 40 -c 1 -o gpurun_out/prof_persist python tools/kprof.py --opt spmv=5 > gpurun_out/prof_persist.log 2>&1
