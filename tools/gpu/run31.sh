#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/pytest31.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest31.log
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --no-gmres > gpurun_out/bench31.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none -c 2000 --csv --log-file gpurun_out/launches31.csv python bench.py --steps 1 --warmup 3 --no-cpu --no-gmres --opt spmv=16 > /dev/null 2>&1
