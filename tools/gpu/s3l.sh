#!/bin/bash
# C3 and C5 bench lines of the current build (GMRES comparator included), C3 launch list
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1200 python bench.py --config C3 --no-cpu > gpurun_out/s3l_bench_C3.log 2>&1; echo "rc=$?" >> gpurun_out/s3l_bench_C3.log
free -g > gpurun_out/s3l_host.txt
timeout 2400 python bench.py --config C5 --steps 3 --warmup 3 --no-cpu > gpurun_out/s3l_bench_C5.log 2>&1; echo "rc=$?" >> gpurun_out/s3l_bench_C5.log
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 3000 --csv --log-file gpurun_out/s3l_launches_C3.csv python bench.py --config C3 --steps 1 --warmup 3 --no-cpu --no-gmres --opt spmv=16 > /dev/null 2>&1
