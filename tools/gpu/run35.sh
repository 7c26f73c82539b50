#!/bin/bash
# round evidence: full GPU suite, smoke, default bench (+cpu), reference arm, launch list, ncu full of the SpMV
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvidia-smi > gpurun_out/smi.txt 2>&1
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/pytest35.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest35.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke35.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke35.log
timeout 900 python bench.py > gpurun_out/bench35.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench35.log
timeout 900 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/bench35_ref.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none -c 2000 --csv --log-file gpurun_out/launches35.csv python bench.py --steps 1 --warmup 3 --no-cpu --no-gmres > /dev/null 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:spmv_dia -s 60 -c 1 -o gpurun_out/prof_spmv35 python tools/kprof.py --opt spmv=16 > /dev/null 2>&1
