#!/bin/bash
# round 2, step A: multi-rank device path through the in-process group + regression suite + bench
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_multirank.py -q -x --durations=15 > gpurun_out/r2a_multirank.log 2>&1; echo "rc=$?" >> gpurun_out/r2a_multirank.log
timeout 1200 python -m pytest tests/test_gpu_parity.py -q --durations=10 > gpurun_out/r2a_parity.log 2>&1; echo "rc=$?" >> gpurun_out/r2a_parity.log
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu > gpurun_out/r2a_bench.log 2>&1; echo "rc=$?" >> gpurun_out/r2a_bench.log
