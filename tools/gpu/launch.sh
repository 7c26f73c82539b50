#!/bin/bash
# launch lists (ncu gpu__time_duration) of one bench solve for several option sets
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
i=0
for o in "$@"; do
  i=$((i+1))
  args=""
  for kv in $o; do args="$args --opt $kv"; done
  timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu $args > gpurun_out/bench_$i.log 2>&1
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$i.csv python bench.py --steps 1 --warmup 3 --no-cpu $args > gpurun_out/ncu_$i.log 2>&1
done
