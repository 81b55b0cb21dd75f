#!/bin/bash
TAG=${1:-r2b}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || { cat gpurun_out/${TAG}_build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_multirank.py tests/test_gpu_graph.py tests/test_gpu_nccl.py -q -rs > gpurun_out/${TAG}_gpu_tests.log 2>&1
tail -n 12 gpurun_out/${TAG}_gpu_tests.log
timeout 600 python tools/growth.py bbh_small_gw bbh5_gw small_gw bbh_small_gw_per > gpurun_out/${TAG}_growth.txt 2>&1
cat gpurun_out/${TAG}_growth.txt
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_case.py 4 > gpurun_out/${TAG}_sanitize_${tool}.txt 2>&1
  tail -n 3 gpurun_out/${TAG}_sanitize_${tool}.txt
done
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
cut -c1-600 gpurun_out/${TAG}_bench.json; tail -3 gpurun_out/${TAG}_bench.err
for c in c1 c2; do timeout 300 python bench.py --config $c --no-cpu-baseline --steps 20 > gpurun_out/${TAG}_bench_$c.json 2>&1; cut -c1-300 gpurun_out/${TAG}_bench_$c.json; done
