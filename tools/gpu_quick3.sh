python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/q_smoke.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multirank.py -x -q > gpurun_out/q_tests.log 2>&1
DGR_FUSED=1 timeout 300 python tools/quick_time.py c3 5 > gpurun_out/q_time_fused.log 2>&1
tail -n 3 gpurun_out/q_smoke.log gpurun_out/q_tests.log; grep -v mesh gpurun_out/q_time_fused.log
