#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "onepass or tsqr_parity or borth or solve_C1 or full_size_C2" > gpurun_out/pytest22.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest22.log
for cfg in "A:" "B:--opt panel_tw=32" "C:--onepass" "D:--onepass --opt panel_tw=32"; do
  tag=${cfg%%:*}; args=${cfg#*:}
  timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu --no-gmres $args > gpurun_out/bench22_$tag.log 2>&1
  timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 1500 --csv --log-file gpurun_out/launches22_$tag.csv python bench.py --steps 1 --warmup 3 --no-cpu --no-gmres --opt spmv=11 $args > /dev/null 2>&1
done
