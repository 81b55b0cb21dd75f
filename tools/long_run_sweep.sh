python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for cfg in "0.4 2.0 0.1" "0.8 2.0 0.25" "0.4 1.0 0.25" "0.1 2.0 0.25" "0.8 1.0 0.1"; do
  set -- $cfg
  DGR_SIGMA=$1 DGR_ETA=$2 DGR_CFL=$3 DGR_BC=somm timeout 200 python tools/long_run.py 24 6 2>&1 | grep -v "^---\|wall"
done > gpurun_out/long_run_sweep.txt
timeout 400 python -m pytest tests/test_gpu_parity.py -x -q -k "unzip or rhs_parity or rk4_step" > gpurun_out/q_tests.log 2>&1
DGR_FUSED=1 timeout 300 python tools/quick_time.py c3 5 > gpurun_out/q_time_fused.log 2>&1
cat gpurun_out/long_run_sweep.txt; tail -n 1 gpurun_out/q_tests.log; grep -v mesh gpurun_out/q_time_fused.log
