#!/bin/bash
# Round-2 session K: full GPU tests (zip owner = coarsest, new golden, new
# k_interp sweeps, 16-B unzip stores), bench, c3big, Table III sweep, ncu.
TAG=${1:-r2k}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1 || { cat gpurun_out/${TAG}_smoke.log; exit 1; }
tail -1 gpurun_out/${TAG}_smoke.log
timeout 1500 python -m pytest tests -m gpu -q -rs -s > gpurun_out/${TAG}_gpu_tests.log 2>&1
grep -E "passed|failed|AMR per-field" gpurun_out/${TAG}_gpu_tests.log | tail -4
timeout 600 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
cut -c1-300 gpurun_out/${TAG}_bench.json; tail -2 gpurun_out/${TAG}_bench.err
timeout 600 python bench.py --config c3big --no-cpu-baseline --steps 10 > gpurun_out/${TAG}_bench_c3big.json 2>&1; cut -c1-300 gpurun_out/${TAG}_bench_c3big.json
timeout 900 python tools/table3_sweep.py 5 > gpurun_out/${TAG}_table3.jsonl 2>&1; cat gpurun_out/${TAG}_table3.jsonl
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_interp|k_unzip" -s 4 -c 3 -o gpurun_out/${TAG}_interp python tools/quick_time.py c3 1 > /dev/null 2>&1
DGR_FUSED=0 timeout 600 ncu --set full --clock-control none -k regex:"k_unzip" -s 1 -c 1 -o gpurun_out/${TAG}_unzip python tools/quick_time.py c3 1 > /dev/null 2>&1
ls gpurun_out/${TAG}_*.ncu-rep
timeout 600 ncu --metrics smsp__sass_thread_inst_executed_op_dfma_pred_on.sum,smsp__sass_thread_inst_executed_op_dadd_pred_on.sum,smsp__sass_thread_inst_executed_op_dmul_pred_on.sum,gpu__time_duration.sum --clock-control none -k regex:"k_rhs|k_gt_pre" -s 8 -c 2 --csv --log-file gpurun_out/${TAG}_flops.csv python tools/quick_time.py c3 1 > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
