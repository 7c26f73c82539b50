#!/bin/bash
# ring SpMV variants: bitwise tests, per-variant timing, bench (autotuned default)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "spmv_variants or mpk_parity or solve_C1 or gmres or tsqr_parity" > gpurun_out/pytest16.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest16.log
timeout 600 python tools/spmv_variants.py > gpurun_out/spmv_variants.json 2> gpurun_out/spmv_variants.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu > gpurun_out/bench16.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench16.log
for v in 10 11 13; do timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu --no-gmres --opt spmv=$v > gpurun_out/bench16_v$v.log 2>&1; done
