python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for cfg in "cell 8 0.4" "cell 8 0.1" "cell 9 0.4" "c2 9 0.4"; do
  set -- $cfg
  DGR_PUNCT=$1 DGR_LMAX=$2 DGR_SIGMA=$3 DGR_BC=somm timeout 400 python tools/long_run.py 40 8 2>&1 | grep -v "^---"
done > gpurun_out/long_run_sweep2.txt
cat gpurun_out/long_run_sweep2.txt
