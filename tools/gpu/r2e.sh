#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
MARGINS_ONLY=C1_svqr,C1_cholqr2,C1_cgs2,C1_mgs,C1_caqr timeout 900 python tools/parity_margins.py > gpurun_out/r2e_margins_variants.json 2> gpurun_out/r2e_margins.err
bash tools/gpu/ncu_panels.sh r2
timeout 900 python bench.py --config C5 --steps 2 --warmup 3 --no-cpu > gpurun_out/r2e_bench_C5.log 2>&1
