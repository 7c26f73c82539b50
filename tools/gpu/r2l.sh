#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_multirank.py -q -k "bench_row_distribution or peer" > gpurun_out/r2l_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r2l_pytest.log
timeout 900 python tools/c4_study.py > gpurun_out/r2l_c4_study.json 2> gpurun_out/r2l_c4_study.err
