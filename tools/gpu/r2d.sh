#!/bin/bash
# round 2, step D: full GPU suite after pruning + early-start ring kernels; bench; panel-kernel ncu
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q -x --durations=10 > gpurun_out/r2d_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r2d_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2d_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/r2d_smoke.log
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu > gpurun_out/r2d_bench.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 2000 --csv --log-file gpurun_out/r2d_launches_C2.csv python bench.py --steps 1 --warmup 3 --no-cpu --no-gmres > /dev/null 2>&1
for k in gram_ring trsm_ring xty_pipe rows_pipe; do
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:$k -s 8 -c 1 -o gpurun_out/r2d_ncu_$k python tools/kprof.py > /dev/null 2>&1
done
timeout 300 ncu --set full --clock-control none --import-source on -k regex:spmv_dia -s 150 -c 1 -o gpurun_out/r2d_ncu_spmv_C3 python tools/kprof.py --config C3 > /dev/null 2>&1
