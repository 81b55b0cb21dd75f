#!/bin/bash
# fresh source-level profile of k_rhs / k_gt_pre / k_interp (product library) + per-stage cycles
TAG=${1:-r3c}
mkdir -p gpurun_out
DGR_LIB=paper_conf_sc_fernandonhzsgb22_b200/lib/libdgr_timing.so timeout 300 python tools/rhs_stage_profile.py c3 > gpurun_out/${TAG}_stage_profile.txt 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"k_rhs|k_gt_pre|k_interp" -s 3 -c 3 -o gpurun_out/${TAG}_full python tools/quick_time.py c3 1 > gpurun_out/${TAG}_ncu.log 2>&1
ls -la gpurun_out
