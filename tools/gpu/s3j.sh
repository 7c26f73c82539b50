#!/bin/bash
# persistent MPK (mpk_wave=3): bitwise tests, C2/C3 bench A/B, MPK-only timing
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest -q -x tests/test_gpu_parity.py -k "sweep or wave or serpentine" > gpurun_out/s3j_tests.log 2>&1; echo "rc=$?" >> gpurun_out/s3j_tests.log
for rep in 1 2; do
  for o in "mpk_wave=3" "mpk_wave=0"; do
    timeout 600 python bench.py --no-cpu --no-gmres --steps 10 --opt $o > gpurun_out/s3j_bench_${rep}_${o}.json 2> gpurun_out/s3j_bench.err
  done
done
for o in "mpk_wave=3" "mpk_wave=0"; do
  timeout 900 python bench.py --config C3 --no-cpu --no-gmres --steps 5 --opt $o > gpurun_out/s3j_C3_${o}.json 2> gpurun_out/s3j_C3.err
done
