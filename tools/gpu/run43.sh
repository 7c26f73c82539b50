#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python tools/tsqr_study.py > gpurun_out/tsqr_study43.json 2> gpurun_out/tsqr_study43.log
timeout 600 python bench.py --config C3 --steps 3 --warmup 3 --no-cpu > gpurun_out/bench43_C3.log 2>&1
