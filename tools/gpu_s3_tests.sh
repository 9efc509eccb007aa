#!/bin/bash
# full-size sampled parity (incl. dmr, amr), then every BASELINE config's bench line
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_amr.py -q -x -k "full_size" --durations=10 > gpurun_out/pytest_full.log 2>&1
echo "pytest full exit $?" >> gpurun_out/pytest_full.log
rm -f gpurun_out/configs.jsonl
for c in sod vortex tgv ramp dmr amr; do
  timeout 900 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 4 >> gpurun_out/configs.jsonl 2>> gpurun_out/configs.err
done
echo done >> gpurun_out/configs.err
