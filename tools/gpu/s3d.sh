#!/bin/bash
# fused residual norm: tests + same-box A/B (exp bit 1 = separate pass); clean-L2 stream calibration
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/sp tools/stream_probe.cu > /dev/null 2>&1
timeout 120 /tmp/sp > gpurun_out/s3d_stream_probe.txt 2>&1
timeout 900 python -m pytest -q -x tests/test_gpu_parity.py -k "solve or normalisation or graph or serp or fold" > gpurun_out/s3d_tests.log 2>&1; echo "rc=$?" >> gpurun_out/s3d_tests.log
for rep in 1 2; do
  for o in "exp=2" "exp=0"; do
    timeout 600 python bench.py --no-cpu --no-gmres --steps 10 --opt $o > gpurun_out/s3d_bench_${rep}_${o}.json 2> gpurun_out/s3d_bench.err
  done
done
timeout 900 python -m pytest -q -x tests/test_gpu_multirank.py tests/test_gpu_numerics.py > gpurun_out/s3d_tests2.log 2>&1; echo "rc=$?" >> gpurun_out/s3d_tests2.log
