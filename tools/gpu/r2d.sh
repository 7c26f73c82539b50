#!/bin/bash
# round 2, step D: full GPU suite after pruning + early-start ring kernels; bench; wave tune
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q --durations=10 > gpurun_out/r2d_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r2d_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2d_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/r2d_smoke.log
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu > gpurun_out/r2d_bench.log 2>&1
timeout 900 python tools/wave_tune.py C2 > gpurun_out/r2d_wave_tune.json 2> gpurun_out/r2d_wave_tune.err
