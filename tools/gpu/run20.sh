#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "onepass or tsqr_parity or borth" > gpurun_out/pytest20.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest20.log
timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu --no-gmres --onepass > gpurun_out/bench20_op.log 2>&1
timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu --no-gmres --onepass --reorth > gpurun_out/bench20_op2.log 2>&1
timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu --no-gmres --reorth > gpurun_out/bench20_2.log 2>&1
