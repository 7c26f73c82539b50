#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "tsqr_parity" > gpurun_out/pytest41.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest41.log
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --no-gmres > gpurun_out/bench41_g1.log 2>&1
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --no-gmres --opt gram=2 > gpurun_out/bench41_g2.log 2>&1
timeout 300 python tools/panel_probe.py > gpurun_out/panel_probe41.json 2> gpurun_out/panel_probe41.log
