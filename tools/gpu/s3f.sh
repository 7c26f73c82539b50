#!/bin/bash
# deeper rings for the 1-4 column Arnoldi / norm passes: tests + A/B (exp bit 3 = old 3-stage rings)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest -q -x tests/test_gpu_parity.py -k "gmres or newton_first or normalisation or graph or clear_shifts" > gpurun_out/s3f_tests.log 2>&1; echo "rc=$?" >> gpurun_out/s3f_tests.log
for rep in 1 2; do
  for o in "exp=8" "exp=0"; do
    timeout 600 python bench.py --no-cpu --no-gmres --steps 10 --opt $o > gpurun_out/s3f_bench_${rep}_${o}.json 2> gpurun_out/s3f_bench.err
  done
done
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 2000 --csv --log-file gpurun_out/s3f_launches_C2.csv python bench.py --steps 1 --warmup 3 --no-cpu --no-gmres > /dev/null 2>&1
