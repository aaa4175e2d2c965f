#!/bin/bash
# Profiling pass for profiles/ (run on the GPU box from the repo root):
#   launch list of rgsqr_factor at BASELINE config 2 (cold-cache, serialised: compare shares) +
#   ncu --set full of the leaf kernel (one plain leaf, one with the folded prologue) and of the
#   top-level K1 / K2 GEMMs.  Summaries: tools/ncu_summary.py, tools/launch_summary.py.
set -x
R=${1:-r02}
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv --log-file gpurun_out/launches_$R.csv \
    python tools/run_c2.py 3 > gpurun_out/launches_$R.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:leaf_kernel -s 64 -c 2 -o gpurun_out/${R}_leaf -f \
    python tools/run_c2.py 2 > gpurun_out/ncu_leaf_$R.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:gemm_tc_kernel -s 92 -c 2 -o gpurun_out/${R}_gemm_top -f \
    python tools/run_c2.py 2 > gpurun_out/ncu_gemm_$R.log 2>&1
ls -la gpurun_out
