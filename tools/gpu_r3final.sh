#!/bin/bash
# Closing run of the round-2 continuation session on the final code: smoke, every
# GPU test, bench (+ size sweep, two-pass), launch list, ncu full of the hot
# kernels with source, a C2 evolution (stability with the new kernels).
TAG=${1:-r3z}
mkdir -p gpurun_out/${TAG}_size_sweep
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1 || { cat gpurun_out/${TAG}_smoke.log; exit 1; }
tail -1 gpurun_out/${TAG}_smoke.log
timeout 1800 python -m pytest tests -m gpu -q -rs -s > gpurun_out/${TAG}_gpu_tests.log 2>&1
grep -E "passed|failed|AMR per-field|SKIPPED" gpurun_out/${TAG}_gpu_tests.log | tail -6
timeout 600 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
cut -c1-300 gpurun_out/${TAG}_bench.json; tail -2 gpurun_out/${TAG}_bench.err
for c in c1 c2 c4 c5 c3big; do timeout 600 python bench.py --config $c --no-cpu-baseline --steps 10 > gpurun_out/${TAG}_size_sweep/$c.json 2>&1; cut -c1-200 gpurun_out/${TAG}_size_sweep/$c.json; done
timeout 600 python bench.py --path two-pass --no-cpu-baseline > gpurun_out/${TAG}_bench_twopass.json 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-options > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_rhs|k_gt_pre|k_interp" -s 6 -c 3 -o gpurun_out/${TAG}_full python tools/quick_time.py c3 1 > gpurun_out/${TAG}_ncu_full.log 2>&1
timeout 600 python tools/evolve.py c2 40 20 > gpurun_out/${TAG}_evolve_c2.txt 2>&1; tail -3 gpurun_out/${TAG}_evolve_c2.txt
ls gpurun_out/${TAG}_full.ncu-rep
