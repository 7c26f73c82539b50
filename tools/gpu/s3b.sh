#!/bin/bash
# serpentine order everywhere: new test, full GPU suite, A/B serp 0/1 on C2, warm-cache DRAM bytes per launch
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python -m pytest -q -x tests/test_gpu_parity.py -k "serpentine or fold or graph or bitwise" > gpurun_out/s3b_tests.log 2>&1; echo "rc=$?" >> gpurun_out/s3b_tests.log
for rep in 1 2; do
  for o in "serp=0" "serp=1"; do
    timeout 600 python bench.py --no-cpu --no-gmres --steps 10 --opt $o > gpurun_out/s3b_bench_${rep}_${o}.json 2> gpurun_out/s3b_bench.err
  done
done
for o in 0 1; do
  timeout 600 ncu --cache-control none --clock-control none --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum -c 1200 --csv --log-file gpurun_out/s3b_warm_serp$o.csv python tools/kprof.py --opt serp=$o > /dev/null 2>&1
done
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/s3b_pytest_all.log 2>&1; echo "rc=$?" >> gpurun_out/s3b_pytest_all.log
