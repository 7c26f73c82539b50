#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest -q -x tests/test_gpu_parity.py -k "solve or normalisation or graph or clear_shifts" > gpurun_out/s3q_tests.log 2>&1; echo "rc=$?" >> gpurun_out/s3q_tests.log
bash tools/gpu/ab.sh norm C2 10 3 "-" "exp=1"
