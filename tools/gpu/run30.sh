#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "tsqr or borth or solve_C1 or gmres or onepass or full_size" > gpurun_out/pytest30.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest30.log
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --no-gmres > gpurun_out/bench30_pf.log 2>&1
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --no-gmres --opt panel_pf=0 > gpurun_out/bench30_nopf.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 2000 --csv --log-file gpurun_out/launches30.csv python bench.py --steps 1 --warmup 3 --no-cpu --no-gmres --opt spmv=16 > /dev/null 2>&1
