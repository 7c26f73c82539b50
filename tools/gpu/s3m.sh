#!/bin/bash
# L2 eviction-priority hints A/B (exp bits 4: update Q evict_first / P evict_last; 5: Gram P evict_last)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python -m pytest -q -x tests/test_gpu_parity.py -k "borth or fold" > gpurun_out/s3m_tests.log 2>&1; echo "rc=$?" >> gpurun_out/s3m_tests.log
for rep in 1 2; do
  for o in "exp=0" "exp=48" "exp=112" "exp=96"; do
    timeout 600 python bench.py --no-cpu --no-gmres --steps 10 --opt $o > gpurun_out/s3m_bench_${rep}_${o}.json 2> gpurun_out/s3m_bench.err
  done
done
for o in "exp=0" "exp=112"; do
  timeout 900 python bench.py --config C3 --no-cpu --no-gmres --steps 5 --opt $o > gpurun_out/s3m_C3_${o}.json 2> gpurun_out/s3m_C3.err
done
timeout 600 ncu --cache-control none --clock-control none --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum -c 1200 --csv --log-file gpurun_out/s3m_warm_exp112.csv python tools/kprof.py --opt spmv=16 --opt exp=112 > /dev/null 2>&1
timeout 600 ncu --cache-control none --clock-control none --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum -c 1200 --csv --log-file gpurun_out/s3m_warm_exp0.csv python tools/kprof.py --opt spmv=16 > /dev/null 2>&1
