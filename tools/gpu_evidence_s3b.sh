#!/bin/bash
# evidence after the xi viscous fusion: launch list of the bench command, full ncu of the stage kernels
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
B="python bench.py --steps 1 --warmup 1 --no-cpu-baseline --e2e-steps 0 --no-clocks"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv $B > gpurun_out/ncu_launch.log 2>&1
export KB_N=512 KB_REPS=1 KB_OVERLAP=0
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"k_sweep|k_visc|k_boxops" -s 7 -c 7 -o gpurun_out/prof_s3 python tools/kbench.py > gpurun_out/ncu_s3.log 2>&1
ncu -i gpurun_out/prof_s3.ncu-rep --page details > gpurun_out/prof_s3_details.txt 2>/dev/null
