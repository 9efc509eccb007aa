cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
B="python bench.py --steps 1 --warmup 1 --no-cpu-baseline --e2e-steps 0 --no-clocks"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv $B > gpurun_out/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_flux -c 3 -o gpurun_out/prof_flux $B > gpurun_out/ncu_flux.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_assemble|k_visc|k_prims" -c 3 -o gpurun_out/prof_other $B > gpurun_out/ncu_other.log 2>&1
ls -la gpurun_out
