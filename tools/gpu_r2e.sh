#!/bin/bash
TAG=${1:-r2e}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || { cat gpurun_out/${TAG}_build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_regrid.py -q -rs > gpurun_out/${TAG}_gpu_tests.log 2>&1; tail -n 3 gpurun_out/${TAG}_gpu_tests.log
DGR_UPWIND=1 DGR_BC=somm timeout 900 python tools/long_run.py 100 40 > gpurun_out/${TAG}_long_upwind_somm.txt 2>&1; cat gpurun_out/${TAG}_long_upwind_somm.txt
DGR_UPWIND=1 DGR_BC=somm DGR_SIGMA=0.1 timeout 900 python tools/long_run.py 100 20 > gpurun_out/${TAG}_long_upwind_somm_s01.txt 2>&1; tail -8 gpurun_out/${TAG}_long_upwind_somm_s01.txt
