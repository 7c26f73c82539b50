#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "spmv or tsqr or kernel_options or fused" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python tools/spmv_variants.py > gpurun_out/spmv_variants.json 2> gpurun_out/spmv_variants.log
timeout 300 python tools/microbench.py > gpurun_out/microbench.json 2>&1
