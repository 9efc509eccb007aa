#!/bin/bash
# round-1 session-3 evidence: default bench (e2e over 16 jobs), reference arm, AMR launch list and
# full ncu of the AMR kernels (k_cf_interp, k_average_down)
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/bench.log 2>&1
echo "bench exit $?" >> gpurun_out/bench.log
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref.log 2>&1
echo "ref exit $?" >> gpurun_out/bench_ref.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_amr.csv python bench.py --config amr --steps 1 --warmup 1 --no-clocks > gpurun_out/ncu_launch_amr.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_cf_interp|k_average_down" -s 3 -c 4 -o gpurun_out/prof_amr python bench.py --config amr --steps 1 --warmup 1 --no-clocks > gpurun_out/ncu_amr.log 2>&1
ncu -i gpurun_out/prof_amr.ncu-rep --page details > gpurun_out/prof_amr_details.txt 2>/dev/null
ncu -i gpurun_out/prof_amr.ncu-rep --page raw --csv > gpurun_out/prof_amr_raw.csv 2>/dev/null
