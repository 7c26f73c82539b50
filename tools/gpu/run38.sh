#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "spmv_variants or mpk_parity or solve_g3" > gpurun_out/pytest38.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest38.log
timeout 600 python tools/spmv_variants.py > gpurun_out/spmv_variants38.json 2> gpurun_out/spmv_variants38.log
timeout 600 python bench.py --config C3 --steps 3 --warmup 3 --no-cpu > gpurun_out/bench38_C3.log 2>&1
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --no-gmres > gpurun_out/bench38.log 2>&1
