#!/bin/bash
# parity margins and the C4 TSQR study with the current build
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1800 python tools/parity_margins.py > gpurun_out/margins.json 2> gpurun_out/margins.err
timeout 900 python tools/c4_study.py > gpurun_out/c4_study.json 2> gpurun_out/c4_study.err
