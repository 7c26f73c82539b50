#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "spmv or mpk" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python tools/spmv_variants.py > gpurun_out/spmv_variants.json 2> gpurun_out/spmv_variants.log
nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/fp64_probe tools/fp64_probe.cu && timeout 120 /tmp/fp64_probe > gpurun_out/fp64_probe.jsonl 2>&1
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu > gpurun_out/bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench.log
