#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/tma_probe tools/tma_probe.cu && timeout 300 /tmp/tma_probe > gpurun_out/tma_probe.log 2>&1
timeout 600 python tools/wave_tune.py > gpurun_out/wave_tune.log 2>&1
timeout 300 python tools/microbench.py > gpurun_out/micro.log 2>&1
timeout 300 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "wave or mpk" > gpurun_out/pytest_gpu.log 2>&1
