cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
export KB_N=512
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_sweep|k_visc|k_prims" -s 5 -c 5 -o gpurun_out/prof_sweep python tools/kbench.py > gpurun_out/ncu_sweep.log 2>&1
ncu -i gpurun_out/prof_sweep.ncu-rep --page source --csv --print-source sass -k regex:k_sweep --launch-count 1 > gpurun_out/sweep0_sass.csv 2>/dev/null
