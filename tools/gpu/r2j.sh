#!/bin/bash
# one-sided peer halo + fused sum/Cholesky (in-process group); full GPU suite; smoke; bench; C3 SpMV ncu
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out /tmp/ncu
timeout 2400 python -m pytest tests -m gpu -q --durations=5 > gpurun_out/r2j_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r2j_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2j_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/r2j_smoke.log
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/r2j_bench.log 2>&1
timeout 900 python bench.py --config C3 --steps 3 --warmup 3 --no-cpu > gpurun_out/r2j_bench_C3.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:spmv_dia -s 60 -c 1 -o /tmp/ncu/spmv_C3 python tools/kprof.py --config C3 --mpk-only > /dev/null 2>&1
ncu -i /tmp/ncu/spmv_C3.ncu-rep --page details > gpurun_out/r2j_ncu_spmv_C3.txt 2>&1
ncu -i /tmp/ncu/spmv_C3.ncu-rep --page raw --csv > gpurun_out/r2j_ncu_spmv_C3_raw.csv 2>&1
