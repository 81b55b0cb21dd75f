#!/bin/bash
# light-field pair stages in k_rhs: parity + timing
TAG=${1:-r2l}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1 || { cat gpurun_out/${TAG}_smoke.log; exit 1; }
tail -1 gpurun_out/${TAG}_smoke.log
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multirank.py tests/test_gpu_graph.py -q -s > gpurun_out/${TAG}_tests.log 2>&1
grep -E "passed|failed|AMR per-field" gpurun_out/${TAG}_tests.log | tail -3
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/${TAG}_bench.json 2>&1
python -c "
import json; d=json.loads(open('gpurun_out/${TAG}_bench.json').read().strip().splitlines()[-1]); print(d['ms_per_step'], {k: round(v['ms_per_launch'],4) for k,v in d['kernels'].items()})"
timeout 600 ncu --metrics smsp__sass_thread_inst_executed_op_dfma_pred_on.sum,smsp__sass_thread_inst_executed_op_dadd_pred_on.sum,smsp__sass_thread_inst_executed_op_dmul_pred_on.sum,gpu__time_duration.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum,smsp__inst_executed.sum --clock-control none -k regex:"k_rhs|k_gt_pre" -s 8 -c 2 --csv --log-file gpurun_out/${TAG}_flops.csv python tools/quick_time.py c3 1 > /dev/null 2>&1
