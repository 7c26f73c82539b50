#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out /tmp/ncu
timeout 600 ncu --set full --clock-control none --import-source on -k regex:spmv -s 175 -c 1 -o /tmp/ncu/spmv_C2 python tools/kprof.py --config C2 --mpk-only > gpurun_out/r2m_ncu.log 2>&1
ncu -i /tmp/ncu/spmv_C2.ncu-rep --page details > gpurun_out/r2m_ncu_spmv_C2.txt 2>&1
ncu -i /tmp/ncu/spmv_C2.ncu-rep --page raw --csv > gpurun_out/r2m_ncu_spmv_C2_raw.csv 2>&1
ncu -i /tmp/ncu/spmv_C2.ncu-rep --page source --csv > gpurun_out/r2m_ncu_spmv_C2_source.csv 2>&1
