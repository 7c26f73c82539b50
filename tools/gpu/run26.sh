#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "spmv_variants or mpk_parity" > gpurun_out/pytest26.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest26.log
timeout 600 python tools/spmv_variants.py > gpurun_out/spmv_variants26.json 2> gpurun_out/spmv_variants26.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu --no-gmres > gpurun_out/bench26.log 2>&1
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --no-gmres --opt spmv=11 > gpurun_out/bench26_v11.log 2>&1
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --no-gmres --opt spmv=14 > gpurun_out/bench26_v14.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:spmv_dia -s 40 -c 1 -o gpurun_out/prof_dia14 python tools/kprof.py --opt spmv=14 > /dev/null 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:spmv_dia -s 40 -c 1 -o gpurun_out/prof_dia11 python tools/kprof.py --opt spmv=11 > /dev/null 2>&1
