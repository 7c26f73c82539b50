#!/bin/bash
# calibration probe; SpMV pre-wait prefetch A/B (exp bit 0) on C2; C3 serp A/B
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/sp tools/stream_probe.cu > /dev/null 2>&1
timeout 120 /tmp/sp > gpurun_out/s3c_stream_probe.txt 2>&1
for rep in 1 2; do
  for o in "exp=0" "exp=1"; do
    timeout 600 python bench.py --no-cpu --no-gmres --steps 10 --opt $o > gpurun_out/s3c_bench_${rep}_${o}.json 2> gpurun_out/s3c_bench.err
  done
done
for o in "serp=0" "serp=1"; do
  timeout 900 python bench.py --config C3 --no-cpu --no-gmres --steps 5 --opt $o > gpurun_out/s3c_C3_${o}.json 2> gpurun_out/s3c_C3.err
done
