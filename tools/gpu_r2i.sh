#!/bin/bash
TAG=${1:-r2i}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
run() { echo "### $*"; env "$@" DGR_BC=somm timeout 600 python tools/long_run.py 40 16; }
{
run DGR_ZIP_COARSEST=1 DGR_SIGMA=0.4
run DGR_ZIP_COARSEST=1 DGR_SIGMA=0.4 DGR_UPWIND=1
} > gpurun_out/${TAG}_sweep.txt 2>&1
cat gpurun_out/${TAG}_sweep.txt
