#!/bin/bash
# ncu --set full of the panel kernels + the C3 SpMV and a C2 launch list; only text summaries
# are kept (the .ncu-rep files are large)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out /tmp/ncu
TAG=${1:-r2}
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 2000 --csv --log-file gpurun_out/${TAG}_launches_C2.csv python bench.py --steps 1 --warmup 3 --no-cpu --no-gmres > /dev/null 2>&1
for k in gram_ring trsm_ring xty_pipe rows_pipe; do
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:$k -s 8 -c 1 -o /tmp/ncu/$k python tools/kprof.py > /dev/null 2>&1
  ncu -i /tmp/ncu/$k.ncu-rep --page details > gpurun_out/${TAG}_ncu_${k}.txt 2>&1
  ncu -i /tmp/ncu/$k.ncu-rep --page raw --csv > gpurun_out/${TAG}_ncu_${k}_raw.csv 2>&1
done
timeout 300 ncu --set full --clock-control none --import-source on -k regex:spmv -s 175 -c 1 -o /tmp/ncu/spmv_C3 python tools/kprof.py --config C3 --mpk-only > /dev/null 2>&1
ncu -i /tmp/ncu/spmv_C3.ncu-rep --page details > gpurun_out/${TAG}_ncu_spmv_C3.txt 2>&1
ncu -i /tmp/ncu/spmv_C3.ncu-rep --page raw --csv > gpurun_out/${TAG}_ncu_spmv_C3_raw.csv 2>&1
