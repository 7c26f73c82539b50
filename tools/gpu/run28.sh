#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "clear_shifts or first_cycle or solve_C1" > gpurun_out/pytest28.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest28.log
timeout 600 python bench.py --steps 5 --warmup 3 > gpurun_out/bench28.log 2>&1
timeout 900 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/bench28_ref.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 2000 --csv --log-file gpurun_out/launches28.csv python bench.py --steps 1 --warmup 3 --no-cpu --no-gmres --opt spmv=11 > /dev/null 2>&1
