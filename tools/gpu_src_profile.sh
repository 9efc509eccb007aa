#!/bin/bash
# source-level ncu of the xi sweep (stall samples per CUDA source line of flux.cuh / weno.cuh)
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
export KB_N=256 KB_REPS=1 KB_OVERLAP=0
timeout 900 ncu --set full --clock-control none --import-source on -k k_sweep_s -s 3 -c 1 -o gpurun_out/prof_src python tools/kbench.py > gpurun_out/ncu_src.log 2>&1
ncu -i gpurun_out/prof_src.ncu-rep --page source --csv --print-source cuda > gpurun_out/sweep0_cuda_src.csv 2>/dev/null
ncu -i gpurun_out/prof_src.ncu-rep --page source --csv --print-source sass > gpurun_out/sweep0_sass_src.csv 2>/dev/null
ls -la gpurun_out/sweep0_*
