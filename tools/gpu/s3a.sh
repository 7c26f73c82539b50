#!/bin/bash
# session 3 A/B: L2 serpentine probe, fold tests, fold / serp A/B on the C2 bench, host gap trace
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/l2p tools/l2_reuse_probe.cu > /dev/null 2>&1
timeout 120 /tmp/l2p > gpurun_out/s3a_l2probe.txt 2>&1
timeout 900 python -m pytest -q -x tests/test_gpu_parity.py -k "fold" > gpurun_out/s3a_fold_tests.log 2>&1; echo "rc=$?" >> gpurun_out/s3a_fold_tests.log
for rep in 1 2; do
  for o in "fold=0" "fold=1" "serp=1" "serp=2" "serp=3"; do
    timeout 600 python bench.py --no-cpu --no-gmres --steps 10 --opt $o > gpurun_out/s3a_bench_${rep}_${o}.json 2> gpurun_out/s3a_bench_${rep}.err
  done
done
CAGMRES_GAPTRACE=1 timeout 600 python bench.py --no-cpu --no-gmres --steps 3 > gpurun_out/s3a_gap.json 2> gpurun_out/s3a_gap.err
