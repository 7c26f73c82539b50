#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "onepass or tsqr or solve or gmres" > gpurun_out/pytest23.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest23.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu > gpurun_out/bench23.log 2>&1
timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu --no-gmres --opt trsm=0 > gpurun_out/bench23_t0.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 1500 --csv --log-file gpurun_out/launches23.csv python bench.py --steps 1 --warmup 3 --no-cpu --no-gmres --opt spmv=11 > /dev/null 2>&1
