#!/bin/bash
# Gram kernel options A/B on C2 / C3 (gram=1 default scalar pairs, 0 DMMA xty SYM, 2 per-warp)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for rep in 1 2; do
  for o in "gram=1" "gram=0" "gram=2"; do
    timeout 600 python bench.py --no-cpu --no-gmres --steps 10 --opt $o > gpurun_out/s3k_bench_${rep}_${o}.json 2> gpurun_out/s3k_bench.err
  done
done
for o in "gram=1" "gram=0" "gram=2"; do
  timeout 900 python bench.py --config C3 --no-cpu --no-gmres --steps 5 --opt $o > gpurun_out/s3k_C3_${o}.json 2> gpurun_out/s3k_C3.err
done
