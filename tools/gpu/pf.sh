#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest -q -x tests/test_gpu_parity.py -k "solve or borth or tsqr or graph or serp" > gpurun_out/pf_tests.log 2>&1; echo "rc=$?" >> gpurun_out/pf_tests.log
bash tools/gpu/ab.sh pf C2 10 3 "-" "panel_pf=1"
bash tools/gpu/ab.sh pf3 C3 5 1 "-" "panel_pf=1"
