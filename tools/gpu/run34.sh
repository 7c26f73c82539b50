#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "spmv_variants" > gpurun_out/pytest34.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest34.log
for v in 16 17 18; do timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --no-gmres --opt spmv=$v > gpurun_out/bench34_v$v.log 2>&1; done
