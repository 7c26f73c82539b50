#!/bin/bash
# fused normalisation (q = w/||w|| inside the consuming SpMV): parity + bitwise + bench
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multirank.py -q -x > gpurun_out/r2g_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r2g_pytest.log
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu > gpurun_out/r2g_bench.log 2>&1
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu --no-gmres --opt fuse=2 > gpurun_out/r2g_bench_nofuse.log 2>&1
