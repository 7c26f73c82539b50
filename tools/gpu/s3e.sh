#!/bin/bash
# xTy exact m-tile count A/B (exp bit 2 = old power-of-two buckets) on C2 and C3; BOrth tests
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest -q -x tests/test_gpu_parity.py -k "borth or solve_C1 or onepass or g3" > gpurun_out/s3e_tests.log 2>&1; echo "rc=$?" >> gpurun_out/s3e_tests.log
for rep in 1 2; do
  for o in "exp=4" "exp=0"; do
    timeout 600 python bench.py --no-cpu --no-gmres --steps 10 --opt $o > gpurun_out/s3e_bench_${rep}_${o}.json 2> gpurun_out/s3e_bench.err
  done
done
for o in "exp=4" "exp=0"; do
  timeout 900 python bench.py --config C3 --no-cpu --no-gmres --steps 5 --opt $o > gpurun_out/s3e_C3_${o}.json 2> gpurun_out/s3e_C3.err
done
