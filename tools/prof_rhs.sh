set -x
python -c "import __graft_entry__ as g; g.build()" || exit 1
python -m paper_conf_sc_fernandonhzsgb22_b200.build --variant timing
DGR_LIB=paper_conf_sc_fernandonhzsgb22_b200/lib/libdgr_timing.so timeout 300 python tools/rhs_stage_profile.py c3 > gpurun_out/stage_profile.txt 2>&1
DGR_FUSED=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_rhs|k_interp" -s 2 -c 2 -o gpurun_out/full_r1d python tools/quick_time.py c3 1 > gpurun_out/ncu_full_r1d.log 2>&1
ncu -i gpurun_out/full_r1d.ncu-rep --page source --csv --print-source=sass -k regex:k_rhs > gpurun_out/rhs_sass.csv 2>&1
ncu -i gpurun_out/full_r1d.ncu-rep --page raw --csv > gpurun_out/full_r1d_raw.csv 2>&1
ls -la gpurun_out
