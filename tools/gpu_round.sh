#!/bin/bash
# One full GPU session: build, GPU tests, bench (fused default + two-pass), launch list,
# ncu --set full of the hot kernels with source, FLOP counters.  Outputs under gpurun_out/.
TAG=${1:-r1e}
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1 || exit 1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/${TAG}_gpu_tests.log 2>&1
timeout 500 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
timeout 500 python bench.py --path two-pass --no-cpu-baseline > gpurun_out/${TAG}_bench_twopass.json 2> gpurun_out/${TAG}_bench_twopass.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
DGR_FUSED=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_rhs|k_gt_pre|k_interp|k_rk4" -s 4 -c 4 -o gpurun_out/${TAG}_full python tools/quick_time.py c3 1 > gpurun_out/${TAG}_ncu_full.log 2>&1
timeout 600 ncu --metrics smsp__sass_thread_inst_executed_op_dfma_pred_on.sum,smsp__sass_thread_inst_executed_op_dadd_pred_on.sum,smsp__sass_thread_inst_executed_op_dmul_pred_on.sum,gpu__time_duration.sum --clock-control none -k regex:"k_rhs|k_gt_pre" -s 4 -c 2 --csv --log-file gpurun_out/${TAG}_flops.csv python tools/quick_time.py c3 1 > /dev/null 2>&1
ncu -i gpurun_out/${TAG}_full.ncu-rep --page source --csv --print-source=cuda,sass -k regex:k_rhs > gpurun_out/${TAG}_rhs_src_sass.csv 2>&1
tail -n 2 gpurun_out/${TAG}_gpu_tests.log; cat gpurun_out/${TAG}_bench.json
