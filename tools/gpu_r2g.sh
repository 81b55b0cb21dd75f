#!/bin/bash
# C2 long-run sweep (is the instability driven by KO at refinement interfaces?),
# upwind parity, quick bench.
TAG=${1:-r2g}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || { cat gpurun_out/${TAG}_build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_parity.py -k "upwind or sommerfeld or fused" -q > gpurun_out/${TAG}_tests.log 2>&1; tail -n 3 gpurun_out/${TAG}_tests.log
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/${TAG}_bench.json 2>&1; cut -c1-300 gpurun_out/${TAG}_bench.json
run() { echo "### $*"; env "$@" DGR_BC=somm timeout 600 python tools/long_run.py 40 16; }
{
run DGR_SIGMA=0.0 DGR_UPWIND=0
run DGR_SIGMA=0.0 DGR_UPWIND=1
run DGR_SIGMA=0.05 DGR_UPWIND=1
run DGR_SIGMA=0.4 DGR_UPWIND=1 DGR_RHO=4.0
run DGR_SIGMA=0.1 DGR_UPWIND=1 DGR_RHO=4.0
} > gpurun_out/${TAG}_sweep.txt 2>&1
cat gpurun_out/${TAG}_sweep.txt
