#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mpk_wave -s 1 -c 1 -o gpurun_out/prof_wave_a python tools/wave_profile.py 1024 2 0 > gpurun_out/ncu_wave_a.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mpk_wave -s 1 -c 1 -o gpurun_out/prof_wave_b python tools/wave_profile.py 512 4 0 > gpurun_out/ncu_wave_b.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:spmv_sell32 -s 5 -c 1 -o gpurun_out/prof_spmv python tools/wave_profile.py 1024 2 0 > gpurun_out/ncu_spmv.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -x -k "solve" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu > gpurun_out/bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench.log
