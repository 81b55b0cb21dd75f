#!/bin/bash
# A/B timing of library variants on C3 (quick_time, per-kernel CUDA events),
# alternating, then the RHS/RK4 parity subset on the product library.
#   tools/gpu_ab.sh TAG lib1 lib2 ...   (lib names: libdgr_<name>.so, "" = product)
TAG=$1; shift
mkdir -p gpurun_out
for rep in 1 2; do
for v in "$@"; do
  f=paper_conf_sc_fernandonhzsgb22_b200/lib/libdgr${v:+_$v}.so
  echo "### ${v:-product} (rep $rep)" >> gpurun_out/${TAG}.txt
  DGR_LIB=$f timeout 300 python tools/quick_time.py ${AB_CFG:-c3} 5 2>&1 | grep -v "^mesh\|^fused" >> gpurun_out/${TAG}.txt
done
done
if [ -z "$AB_NOTEST" ]; then
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "${AB_TESTS:-rhs_parity or two_pass or prepass or zip_store or amr or rk4_step_parity}" > gpurun_out/${TAG}_tests.log 2>&1; tail -n 3 gpurun_out/${TAG}_tests.log >> gpurun_out/${TAG}.txt
fi
cat gpurun_out/${TAG}.txt
