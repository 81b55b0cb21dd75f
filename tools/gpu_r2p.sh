#!/bin/bash
# A/B: bank-interleaved gather order vs the source-sorted order
TAG=${1:-r2p}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "rhs_parity or two_pass or prepass or zip_store or amr_golden or rk4_step_parity or constraints" > gpurun_out/${TAG}_tests.log 2>&1; tail -n 2 gpurun_out/${TAG}_tests.log
for v in 1 0 1 0; do
  DGR_GATHER_SORT_ONLY=$v timeout 300 python bench.py --no-cpu-baseline --steps 20 > gpurun_out/${TAG}_bench_sortonly$v.json 2>&1
  python -c "
import json; d=json.loads(open('gpurun_out/${TAG}_bench_sortonly$v.json').read().strip().splitlines()[-1]); print('sort_only=$v', d['ms_per_step'], {k: round(v['ms_per_launch'],4) for k,v in d['kernels'].items()})"
done
for v in 0 1; do
DGR_GATHER_SORT_ONLY=$v timeout 600 ncu --metrics l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ldgsts.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum,gpu__time_duration.sum,lts__t_sectors_srcunit_tex.sum --clock-control none -k regex:"k_rhs|k_gt_pre" -s 8 -c 2 --csv --log-file gpurun_out/${TAG}_ncu_sortonly$v.csv python tools/quick_time.py c3 1 > /dev/null 2>&1
done
grep -h "ldgsts\|gpu__time\|wavefronts\|lts__t" gpurun_out/${TAG}_ncu_sortonly*.csv | cut -d, -f5,13-16 | head -20
