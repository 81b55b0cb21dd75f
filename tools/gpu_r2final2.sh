#!/bin/bash
# Round-2 closing session on the final code: smoke, every GPU test, bench (+ sweep),
# sanitizers, launch list, ncu full summary, FLOPs.
TAG=${1:-r2y}
mkdir -p gpurun_out/${TAG}_size_sweep
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1 || { cat gpurun_out/${TAG}_smoke.log; exit 1; }
tail -1 gpurun_out/${TAG}_smoke.log
timeout 1800 python -m pytest tests -m gpu -q -rs -s > gpurun_out/${TAG}_gpu_tests.log 2>&1
grep -E "passed|failed|AMR per-field|SKIPPED" gpurun_out/${TAG}_gpu_tests.log | tail -6
timeout 600 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
cut -c1-300 gpurun_out/${TAG}_bench.json; tail -2 gpurun_out/${TAG}_bench.err
for c in c1 c2 c4 c5 c3big; do timeout 600 python bench.py --config $c --no-cpu-baseline --steps 10 > gpurun_out/${TAG}_size_sweep/$c.json 2>&1; cut -c1-200 gpurun_out/${TAG}_size_sweep/$c.json; done
timeout 600 python bench.py --path two-pass --no-cpu-baseline > gpurun_out/${TAG}_bench_twopass.json 2>&1
for tool in memcheck racecheck synccheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_case.py 4 > gpurun_out/${TAG}_sanitize_${tool}.txt 2>&1
  tail -n 2 gpurun_out/${TAG}_sanitize_${tool}.txt
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_rhs|k_gt_pre|k_interp|k_rk4" -s 8 -c 4 -o gpurun_out/${TAG}_full python tools/quick_time.py c3 1 > gpurun_out/${TAG}_ncu_full.log 2>&1
timeout 600 ncu --metrics smsp__sass_thread_inst_executed_op_dfma_pred_on.sum,smsp__sass_thread_inst_executed_op_dadd_pred_on.sum,smsp__sass_thread_inst_executed_op_dmul_pred_on.sum,gpu__time_duration.sum --clock-control none -k regex:"k_rhs|k_gt_pre" -s 8 -c 2 --csv --log-file gpurun_out/${TAG}_flops.csv python tools/quick_time.py c3 1 > /dev/null 2>&1
ls gpurun_out/${TAG}_full.ncu-rep
