#!/bin/bash
TAG=${1:-r2h}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
DGR_RHO=1.0 timeout 600 python tools/instab_probe.py > gpurun_out/${TAG}_probe_rho1.txt 2>&1; cat gpurun_out/${TAG}_probe_rho1.txt
DGR_RHO=4.0 timeout 900 python tools/instab_probe.py > gpurun_out/${TAG}_probe_rho4.txt 2>&1; cat gpurun_out/${TAG}_probe_rho4.txt
