#!/bin/bash
# C5 (BASELINE.json's large config, 27-pt 400^3, n = 64M, 1.72e9 nnz) on one B200: complete
# solves timed by bench.py.  Host needs ~50 GB (CSR 21 GB + generator temporaries + setup copies).
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
free -g > gpurun_out/c5_host.txt; nproc >> gpurun_out/c5_host.txt
avail=$(free -g | awk '/Mem:/{print $7}')
if [ "$avail" -lt 120 ]; then echo "host memory too small: ${avail} GB" > gpurun_out/bench_C5.log; exit 0; fi
timeout 1500 python bench.py --config C5 --steps 3 --warmup 3 --no-cpu --no-gmres > gpurun_out/bench_C5.log 2>&1
echo "bench rc=$?" >> gpurun_out/bench_C5.log
