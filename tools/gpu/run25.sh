#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/pytest25.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest25.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu > gpurun_out/bench25.log 2>&1
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --no-gmres --opt pdl=0 > gpurun_out/bench25_nopdl.log 2>&1
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --no-gmres --opt trsm=0 > gpurun_out/bench25_t0.log 2>&1
