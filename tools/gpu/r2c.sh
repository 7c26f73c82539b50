#!/bin/bash
# round 2, step C: TMA-streamed SpMV (variants 21/22): bitwise, bench, ncu
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "spmv_variants or mpk_parity or mpk_full_size_C2" > gpurun_out/r2c_variants.log 2>&1; echo "rc=$?" >> gpurun_out/r2c_variants.log
for v in 16 21 22; do
  timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu --no-gmres --opt spmv=$v > gpurun_out/r2c_bench_spmv$v.log 2>&1
done
timeout 300 python bench.py --config C5 --steps 2 --warmup 3 --no-cpu --no-gmres --opt spmv=21 > gpurun_out/r2c_bench_C5_spmv21.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:spmv_tma -s 60 -c 1 -o gpurun_out/r2c_ncu_spmv_tma python tools/kprof.py --opt spmv=21 > gpurun_out/r2c_ncu.log 2>&1
