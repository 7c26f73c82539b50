#!/bin/bash
# round evidence: full GPU suite, smoke, default bench (+cpu), reference arm, launch list,
# ncu --set full of the dominant kernel (MPK SpMV, variant 16)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvidia-smi > gpurun_out/smi.txt 2>&1
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_final.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_final.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_final.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke_final.log
timeout 900 python bench.py > gpurun_out/bench_final.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench_final.log
timeout 900 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/bench_ref_final.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none -c 2000 --csv --log-file gpurun_out/launches_final.csv python bench.py --steps 1 --warmup 3 --no-cpu --no-gmres --opt spmv=16 > /dev/null 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:"spmv_dia" -s 400 -c 1 -o gpurun_out/prof_spmv_final python tools/kprof.py --opt spmv=16 > /dev/null 2>&1
