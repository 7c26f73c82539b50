#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 python tools/panel_probe.py > gpurun_out/panel_probe.json 2> gpurun_out/panel_probe.log
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches24.csv python tools/panel_probe.py > /dev/null 2>&1
