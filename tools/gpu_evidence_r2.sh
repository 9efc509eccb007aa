#!/bin/bash
# round-2 evidence: GPU tests, smoke, default bench (cpu_baseline suite), reference arm, ncu launch
# list of one bench step and a full ncu capture of the sweeps + viscous kernel (profiles/).
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
TAG=${TAG:-r02}
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1
echo "smoke exit $?" >> gpurun_out/${TAG}_smoke.log
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/${TAG}_gputest.log 2>&1
echo "pytest exit $?" >> gpurun_out/${TAG}_gputest.log
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/${TAG}_bench.jsonl 2> gpurun_out/${TAG}_bench.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/${TAG}_bench_reference.jsonl 2> gpurun_out/${TAG}_bench_reference.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-clocks --e2e-steps 0 > gpurun_out/${TAG}_ncu_launch.log 2>&1
if [ -n "$FULL" ]; then
  KB_REPS=1 KB_OVERLAP=0 timeout 1200 ncu --set full --import-source on --clock-control none \
    -k regex:"k_sweep_s|k_visc_tiled|k_fill_gather" -s 5 -c 5 -o gpurun_out/${TAG}_kernels -f python tools/kbench.py > gpurun_out/${TAG}_ncu_full.log 2>&1
fi
