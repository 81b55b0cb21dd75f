#!/bin/bash
TAG=${1:-r2d}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || { cat gpurun_out/${TAG}_build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_regrid.py "tests/test_gpu_parity.py::test_100_steps_amr_golden" -q -s -rs > gpurun_out/${TAG}_gpu_tests.log 2>&1
tail -n 25 gpurun_out/${TAG}_gpu_tests.log
timeout 900 ncu --metrics smsp__sass_thread_inst_executed_op_dfma_pred_on.sum,smsp__sass_thread_inst_executed_op_dadd_pred_on.sum,smsp__sass_thread_inst_executed_op_dmul_pred_on.sum,gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active,launch__registers_per_thread --clock-control none -k regex:"k_alg|k_rhs_inputs|k_rhs|k_gt_pre" -c 24 --csv --log-file gpurun_out/${TAG}_codegen_ncu.csv python tools/codegen_bench.py c2 1 > /dev/null 2>&1
wc -l gpurun_out/${TAG}_codegen_ncu.csv
