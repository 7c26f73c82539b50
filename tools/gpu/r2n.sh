#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "variants or fused or mpk_parity" > gpurun_out/r2n_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r2n_pytest.log
timeout 900 python tools/spmv_variants.py > gpurun_out/r2n_spmv_variants.json 2> gpurun_out/r2n_spmv_variants.err
for v in 16 18 19; do timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu --no-gmres --opt spmv=$v > gpurun_out/r2n_bench_spmv$v.log 2>&1; done
