#!/bin/bash
# C3 and C5 bench lines (GMRES comparator included) of the current build
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1200 python bench.py --config C3 --no-cpu > gpurun_out/c35_bench_C3.log 2>&1; echo "rc=$?" >> gpurun_out/c35_bench_C3.log
timeout 2400 python bench.py --config C5 --steps 3 --warmup 3 --no-cpu > gpurun_out/c35_bench_C5.log 2>&1; echo "rc=$?" >> gpurun_out/c35_bench_C5.log
