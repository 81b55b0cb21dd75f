#!/bin/bash
# Round-2 GPU session A: build, smoke, GPU tests, growth study for the AMR
# 100-step parity case, compute-sanitizer, bench.  Outputs under gpurun_out/.
TAG=${1:-r2a}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1 || { cat gpurun_out/${TAG}_smoke.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/${TAG}_gpu_tests.log 2>&1
tail -n 15 gpurun_out/${TAG}_gpu_tests.log
timeout 900 python tools/growth.py bbh_small bbh_small_rand bbh5_bl bbh5_rand small_bl small_rand > gpurun_out/${TAG}_growth.txt 2>&1
cat gpurun_out/${TAG}_growth.txt
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_case.py 4 > gpurun_out/${TAG}_sanitize_${tool}.txt 2>&1
  tail -n 3 gpurun_out/${TAG}_sanitize_${tool}.txt
done
timeout 600 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
cat gpurun_out/${TAG}_bench.json
