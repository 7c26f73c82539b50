#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "borth or solve or onepass" > gpurun_out/pytest40.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest40.log
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --no-gmres > gpurun_out/bench40.log 2>&1
timeout 600 python bench.py --config C3 --steps 3 --warmup 3 --no-cpu --no-gmres > gpurun_out/bench40_C3.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none -c 2000 --csv --log-file gpurun_out/launches40.csv python bench.py --steps 1 --warmup 3 --no-cpu --no-gmres > /dev/null 2>&1
