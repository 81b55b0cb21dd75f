#!/bin/bash
TAG=${1:-r2m}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || { cat gpurun_out/${TAG}_build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_psi4.py tests/test_gpu_codegen.py tests/test_gpu_regrid.py -q -rs > gpurun_out/${TAG}_tests.log 2>&1; tail -n 15 gpurun_out/${TAG}_tests.log
