#!/bin/bash
TAG=${1:-r2j}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
{
echo "### C2, both outer boundaries, KO 0.4, centred advection (defaults), t = 100 M"
timeout 900 python tools/long_run.py 100 40
echo "### C2, Sommerfeld, lopsided advection (R9u), t = 100 M"
DGR_UPWIND=1 DGR_BC=somm timeout 900 python tools/long_run.py 100 20
echo "### C2 finest level 9, Sommerfeld, t = 60 M"
DGR_LMAX=9 DGR_BC=somm timeout 900 python tools/long_run.py 60 12
echo "### C3 (BL q=1 BBH, 24k octants), Sommerfeld, t = 20 M"
DGR_CFG=c3 DGR_BC=somm timeout 1200 python tools/long_run.py 20 10
} > gpurun_out/${TAG}_long.txt 2>&1
cat gpurun_out/${TAG}_long.txt
