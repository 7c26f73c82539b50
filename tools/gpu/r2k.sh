#!/bin/bash
# CUDA-graph CA cycles + xty split accumulators: tests + bench A/B
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out /tmp/ncu
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -x -k "graph or fused or solve or tsqr or borth" > gpurun_out/r2k_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r2k_pytest.log
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu > gpurun_out/r2k_bench.log 2>&1
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu --no-gmres --opt graph=1 > gpurun_out/r2k_bench_graph.log 2>&1
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu --no-gmres > gpurun_out/r2k_bench2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spmv -s 175 -c 1 -o /tmp/ncu/spmv_C3 python tools/kprof.py --config C3 --mpk-only > gpurun_out/r2k_ncu_C3.log 2>&1
ncu -i /tmp/ncu/spmv_C3.ncu-rep --page details > gpurun_out/r2k_ncu_spmv_C3.txt 2>&1
ncu -i /tmp/ncu/spmv_C3.ncu-rep --page raw --csv > gpurun_out/r2k_ncu_spmv_C3_raw.csv 2>&1
