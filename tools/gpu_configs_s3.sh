#!/bin/bash
# every bench config after the xi viscous fusion
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
: > gpurun_out/configs.jsonl
for c in sod vortex tgv ramp dmr amr dmr_amr; do
  timeout 900 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 4 >> gpurun_out/configs.jsonl 2>> gpurun_out/configs.err
done
echo done >> gpurun_out/configs.err
