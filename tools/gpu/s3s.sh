#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest -q -x tests/test_gpu_parity.py -k "borth or solve or graph or fold or serp" > gpurun_out/s3s_tests.log 2>&1; echo "rc=$?" >> gpurun_out/s3s_tests.log
timeout 900 python -m pytest -q -x tests/test_gpu_multirank.py -k "solve" > gpurun_out/s3s_tests2.log 2>&1; echo "rc=$?" >> gpurun_out/s3s_tests2.log
bash tools/gpu/ab.sh early3 C3 5 2 "-" "exp=2"
bash tools/gpu/ab.sh early2 C2 10 2 "-" "exp=2"
