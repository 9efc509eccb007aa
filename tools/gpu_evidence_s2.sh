# round-1 session-2 evidence: NCCL 2-ranks-on-1-GPU probe, bench (default + reference arm),
# launch list, full ncu of sweeps / viscous / fill, SASS source page of the sweeps
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 240 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 tests/nccl_two_ranks_one_gpu.py > gpurun_out/nccl2.log 2>&1
echo "nccl2 exit $?" >> gpurun_out/nccl2.log
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/bench.log 2>&1
echo "bench exit $?" >> gpurun_out/bench.log
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref.log 2>&1
B="python bench.py --steps 1 --warmup 1 --no-cpu-baseline --e2e-steps 0 --no-clocks"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv $B > gpurun_out/ncu_launch.log 2>&1
export KB_N=512 KB_REPS=1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"k_sweep|k_visc|k_boxops" -s 7 -c 7 -o gpurun_out/prof_s2 python tools/kbench.py > gpurun_out/ncu_s2.log 2>&1
ncu -i gpurun_out/prof_s2.ncu-rep --page source --csv --print-source sass -k regex:"k_sweep_s<1" --launch-count 1 > gpurun_out/sweep1_s2_sass.csv 2>/dev/null
ncu -i gpurun_out/prof_s2.ncu-rep --page details > gpurun_out/prof_s2_details.txt 2>/dev/null
