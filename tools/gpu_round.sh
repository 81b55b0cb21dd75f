#!/bin/bash
# One GPU session: build, bench both paths, launch list + ncu --set full of the hot kernels.
set -x
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 500 python bench.py --path fused > gpurun_out/bench_fused.json 2> gpurun_out/bench_fused.err
timeout 500 python bench.py --path two-pass --no-cpu-baseline > gpurun_out/bench_twopass.json 2> gpurun_out/bench_twopass.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_fused.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --path fused > /dev/null 2>&1
DGR_FUSED=1 timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_rhs|k_interp|k_zip_rk4" -s 4 -c 3 -o gpurun_out/full_fused python tools/quick_time.py c3 1 > gpurun_out/ncu_full_fused.log 2>&1
DGR_FUSED=0 timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_rhs|k_unzip" -s 4 -c 2 -o gpurun_out/full_twopass python tools/quick_time.py c3 1 > gpurun_out/ncu_full_twopass.log 2>&1
for P in 1 0; do
DGR_FUSED=$P timeout 600 ncu --metrics smsp__sass_thread_inst_executed_op_dfma_pred_on.sum,smsp__sass_thread_inst_executed_op_dadd_pred_on.sum,smsp__sass_thread_inst_executed_op_dmul_pred_on.sum,gpu__time_duration.sum --clock-control none -k regex:"k_rhs" -s 2 -c 1 --csv --log-file gpurun_out/flops_fused$P.csv python tools/quick_time.py c3 1 > /dev/null 2>&1
done
ls -la gpurun_out/
