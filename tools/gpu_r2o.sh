#!/bin/bash
# head-on BL q=1 (C3) waveform: Psi_4 (2,0) and (2,2) modes at r = 40 to t = 120 M
TAG=${1:-r2o}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
DGR_FR=100000000 DGR_EXTRACT=32 timeout 2400 python tools/evolve.py c3 120 40 > gpurun_out/${TAG}_waveform_c3.txt 2>&1
tail -5 gpurun_out/${TAG}_waveform_c3.txt
