#!/bin/bash
TAG=${1:-r2n}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
python -c "from paper_conf_sc_fernandonhzsgb22_b200 import build as b; b.build(variant='timing')" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "unzip or rhs_parity or two_pass or amr_golden" > gpurun_out/${TAG}_tests.log 2>&1; tail -n 2 gpurun_out/${TAG}_tests.log
DGR_LIB=paper_conf_sc_fernandonhzsgb22_b200/lib/libdgr_timing.so timeout 300 python tools/rhs_stage_profile.py c3 > gpurun_out/${TAG}_stage_cycles.txt 2>&1; cat gpurun_out/${TAG}_stage_cycles.txt
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/${TAG}_bench.json 2>&1
python -c "
import json; d=json.loads(open('gpurun_out/${TAG}_bench.json').read().strip().splitlines()[-1]); print(d['ms_per_step'], {k: round(v['ms_per_launch'],4) for k,v in d['kernels'].items()})"
timeout 300 python tools/table3_sweep.py 5 > gpurun_out/${TAG}_table3.jsonl 2>&1; head -1 gpurun_out/${TAG}_table3.jsonl | cut -c1-300
