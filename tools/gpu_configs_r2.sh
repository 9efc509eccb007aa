#!/bin/bash
# round 2: every bench config once (one GPU), plus the slow overlap-depth test
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
: > gpurun_out/configs_r2.jsonl
for cfg in sod vortex tgv ramp dmr amr dmr_amr; do
  timeout 900 python bench.py --config $cfg --steps 5 --warmup 3 --no-cpu-baseline >> gpurun_out/configs_r2.jsonl 2>> gpurun_out/configs_r2.err
done
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "interior_slabs" > gpurun_out/r02_slab.log 2>&1
