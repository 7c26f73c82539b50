#!/bin/bash
# TRSM with R^{-1} in registers (2 rows / lane), update ring stride TW+4: parity + bench + ncu
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out /tmp/ncu
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multirank.py -q -x -k "tsqr or borth or solve or onepass" > gpurun_out/r2f_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r2f_pytest.log
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu > gpurun_out/r2f_bench.log 2>&1
for k in trsm_ring rows_pipe; do
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:$k -s 8 -c 1 -o /tmp/ncu/$k python tools/kprof.py > /dev/null 2>&1
  ncu -i /tmp/ncu/$k.ncu-rep --page details > gpurun_out/r2f_ncu_${k}.txt 2>&1
  ncu -i /tmp/ncu/$k.ncu-rep --page raw --csv > gpurun_out/r2f_ncu_${k}_raw.csv 2>&1
done
