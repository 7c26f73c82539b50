#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "tsqr or solve_C1 or full_size_C2" > gpurun_out/pytest19.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest19.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu --no-gmres > gpurun_out/bench19.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench19.log
timeout 300 ncu --set full --clock-control none --import-source on -k regex:gram_ring -s 6 -c 1 -o gpurun_out/prof_gram64 python tools/kprof.py > gpurun_out/prof_gram.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:rows_pipe -s 40 -c 6 -o gpurun_out/prof_rows2 python tools/kprof.py > gpurun_out/prof_rows.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:xty_pipe -s 10 -c 2 -o gpurun_out/prof_xty2 python tools/kprof.py > gpurun_out/prof_xty.log 2>&1
