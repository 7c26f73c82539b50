#!/bin/bash
# round 2, step B: new numerics tests, parity margins, SpMV L2-hint variants
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_numerics.py -q --durations=20 > gpurun_out/r2b_numerics.log 2>&1; echo "rc=$?" >> gpurun_out/r2b_numerics.log
timeout 600 python -m pytest tests/test_gpu_parity.py -q -k "spmv_variants" > gpurun_out/r2b_variants.log 2>&1; echo "rc=$?" >> gpurun_out/r2b_variants.log
for v in 16 19 20; do
  timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu --no-gmres --opt spmv=$v > gpurun_out/r2b_bench_spmv$v.log 2>&1
done
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:spmv -c 300 --csv --log-file gpurun_out/r2b_launch_spmv19.csv python tools/kprof.py --opt spmv=19 > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:spmv -c 300 --csv --log-file gpurun_out/r2b_launch_spmv16.csv python tools/kprof.py --opt spmv=16 > /dev/null 2>&1
timeout 1500 python tools/parity_margins.py > gpurun_out/r2b_parity_margins.json 2> gpurun_out/r2b_parity_margins.err
