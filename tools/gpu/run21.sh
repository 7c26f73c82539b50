#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 1500 --csv --log-file gpurun_out/launches21.csv python bench.py --steps 1 --warmup 3 --no-cpu --no-gmres --onepass --opt spmv=11 > gpurun_out/ncu_launch21.log 2>&1
