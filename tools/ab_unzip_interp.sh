#!/bin/bash
# A/B of k_unzip loads-in-flight / min-blocks and k_interp CTA size (experiment
# builds lib/libdgr_exp*.so, DGR_LIB selects the library); Table III m1 = C3.
TAG=${1:-r2ab}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
run() {
  v=$1; shift
  DGR_EXTRA_DEFS="$*" python -c "from paper_conf_sc_fernandonhzsgb22_b200 import build as b; b.build(variant='$v')" > /dev/null 2>&1 || { echo "build $v failed"; return; }
  echo "### $v: $*"
  DGR_LIB=paper_conf_sc_fernandonhzsgb22_b200/lib/libdgr_$v.so timeout 300 python tools/table3_sweep.py 5 2>&1 | head -1 | cut -c1-400
}
{
run exp0
run exp1 -DDGR_UZ_U=12 -DDGR_UZ_MINB=4
run exp6 -DDGR_UZ_U=12 -DDGR_UZ_MINB=5
run exp7 -DDGR_UZ_U=14 -DDGR_UZ_MINB=4
run exp8 -DDGR_UZ_U=10 -DDGR_UZ_MINB=5
run exp9 -DDGR_IP_THREADS=128 -DDGR_IP_FG=2
run exp10 -DDGR_IP_THREADS=192
} > gpurun_out/${TAG}.txt 2>&1
cat gpurun_out/${TAG}.txt
