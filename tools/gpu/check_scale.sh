#!/bin/bash
# scale kernel change: parity tests that reach it, then the default C2 bench line
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x -k "tsqr_parity or solve or smoke" > gpurun_out/pytest_scale.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_scale.log
timeout 600 python bench.py > gpurun_out/bench_scale.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench_scale.log
