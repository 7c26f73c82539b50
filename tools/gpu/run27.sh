#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/pytest27.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest27.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke27.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke27.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu > gpurun_out/bench27.log 2>&1
