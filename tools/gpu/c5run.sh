#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -q -x -k "spmv or mpk or solve" > gpurun_out/pytest_spmv.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_spmv.log
bash tools/gpu/c5.sh
