# quick GPU check: smoke, RHS/RK4 parity subset, C3 timings of both paths, per-stage cycle profile
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/q_smoke.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "rhs or rk4 or minkowski or fused" > gpurun_out/q_tests.log 2>&1
DGR_FUSED=1 timeout 300 python tools/quick_time.py c3 5 > gpurun_out/q_time_fused.log 2>&1
DGR_FUSED=0 timeout 300 python tools/quick_time.py c3 5 > gpurun_out/q_time_twopass.log 2>&1
python -m paper_conf_sc_fernandonhzsgb22_b200.build --variant timing > /dev/null
DGR_LIB=paper_conf_sc_fernandonhzsgb22_b200/lib/libdgr_timing.so timeout 300 python tools/rhs_stage_profile.py c3 > gpurun_out/q_stage_profile.txt 2>&1
tail -n 2 gpurun_out/q_smoke.log gpurun_out/q_tests.log; cat gpurun_out/q_time_fused.log gpurun_out/q_time_twopass.log | grep -v mesh; cat gpurun_out/q_stage_profile.txt
