#!/bin/bash
# GMRES baseline parity + bench with the comparator; ncu --set full of SpMV (variant 5) and Gram
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "gmres" > gpurun_out/pytest_gmres.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gmres.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu > gpurun_out/bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench.log
timeout 300 ncu --set full --clock-control none --import-source on -k regex:spmv_sell32_persist -s 60 -c 1 -o gpurun_out/prof_spmv python tools/kprof.py > gpurun_out/prof_spmv.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:gram_ring -s 6 -c 1 -o gpurun_out/prof_gram python tools/kprof.py > gpurun_out/prof_gram.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:rows_pipe -s 20 -c 3 -o gpurun_out/prof_rows python tools/kprof.py > gpurun_out/prof_rows.log 2>&1
