#!/bin/bash
# C5 launch list (SpMV variant pinned, see profiles/README.md) + C2 launch list with the pinned variant
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -s 330 -c 1500 --csv --log-file gpurun_out/launches_C5.csv python bench.py --config C5 --steps 1 --warmup 3 --no-cpu --no-gmres --opt spmv=16 > gpurun_out/launches_C5.log 2>&1
echo "rc=$?" >> gpurun_out/launches_C5.log
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none -s 330 -c 2000 --csv --log-file gpurun_out/launches_final.csv python bench.py --steps 1 --warmup 3 --no-cpu --no-gmres --opt spmv=16 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"spmv_dia" -s 200 -c 1 -o gpurun_out/prof_spmv_C5 python bench.py --config C5 --steps 1 --warmup 3 --no-cpu --no-gmres --opt spmv=16 > /dev/null 2>&1
