#!/bin/bash
# round evidence for the current build: full GPU suite, smoke, default C2 bench (+ oracle
# cpu_baseline, GMRES comparator), reference arm, launch list (SpMV variant pinned to the one the
# bench picks: ncu's serialised replay skews the create-time autotune), ncu --set full of the
# dominant kernel (MPK SpMV) and the panel kernels (text summaries + source page of the Gram).
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out /tmp/ncu
T=${1:-final}
nvidia-smi > gpurun_out/${T}_smi.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/${T}_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${T}_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${T}_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/${T}_smoke.log
timeout 900 python bench.py > gpurun_out/${T}_bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/${T}_bench.log
timeout 900 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/${T}_bench_ref.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 2000 --csv --log-file gpurun_out/${T}_launches_C2.csv python bench.py --steps 1 --warmup 3 --no-cpu --no-gmres --opt spmv=16 > /dev/null 2>&1
for k in spmv_dia gram_ring trsm_ring xty_pipe rows_pipe; do
  s=8; [ $k = spmv_dia ] && s=400
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:$k -s $s -c 1 -o /tmp/ncu/$k python tools/kprof.py --opt spmv=16 > /dev/null 2>&1
  ncu -i /tmp/ncu/$k.ncu-rep --page details > gpurun_out/${T}_ncu_${k}.txt 2>&1
  ncu -i /tmp/ncu/$k.ncu-rep --page raw --csv > gpurun_out/${T}_ncu_${k}_raw.csv 2>&1
done
ncu -i /tmp/ncu/gram_ring.ncu-rep --page source --csv > gpurun_out/${T}_ncu_gram_ring_source.csv 2>&1
