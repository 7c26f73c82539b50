#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "solve or gmres or clear" > gpurun_out/pytest39.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest39.log
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu > gpurun_out/bench39.log 2>&1
