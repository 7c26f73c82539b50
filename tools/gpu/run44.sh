#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "svqr or tsqr_parity or solve_C1" > gpurun_out/pytest44.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest44.log
timeout 900 python tools/tsqr_study.py > gpurun_out/tsqr_study44.json 2> gpurun_out/tsqr_study44.log
