cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
export KB_N=512
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_visc" -s 1 -c 1 -o gpurun_out/prof_visc python tools/kbench.py > gpurun_out/ncu_visc.log 2>&1
