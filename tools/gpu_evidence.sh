# round evidence: bench line (default + reference arm), launch list, full ncu of the hot kernels, configs
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/bench.log 2>&1
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref.log 2>&1
B="python bench.py --steps 1 --warmup 1 --no-cpu-baseline --e2e-steps 0 --no-clocks"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv $B > gpurun_out/ncu_launch.log 2>&1
export KB_N=512 KB_REPS=1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_sweep|k_visc|k_boxops" -s 8 -c 7 -o gpurun_out/prof_final python tools/kbench.py > gpurun_out/ncu_final.log 2>&1
ncu -i gpurun_out/prof_final.ncu-rep --page source --csv --print-source sass -k regex:k_sweep --launch-count 1 > gpurun_out/sweep_final_sass.csv 2>/dev/null
bash tools/gpu_configs.sh
