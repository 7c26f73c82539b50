#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "spmv_variants or mpk or solve or gmres" > gpurun_out/pytest18.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest18.log
timeout 600 python tools/spmv_variants.py > gpurun_out/spmv_variants.json 2> gpurun_out/spmv_variants.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu > gpurun_out/bench18.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench18.log
timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu --no-gmres --opt fuse=3 > gpurun_out/bench18_fuse3.log 2>&1
timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu --opt arnoldi=0 > gpurun_out/bench18_arn0.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file gpurun_out/launches18.csv python bench.py --steps 1 --warmup 3 --no-cpu > gpurun_out/ncu_launch18.log 2>&1
