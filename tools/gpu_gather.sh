#!/bin/bash
# single-pass gather fill: GPU suite, then small-config bench lines and 512^3 stage timing (3-phase vs gather)
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest exit $?" >> gpurun_out/pytest_gpu.log
: > gpurun_out/gather_configs.jsonl
for lib in nogather gather; do
  for c in sod vortex; do
    CROCCO_LIB=$PWD/build/variants/libcrocco_$lib.so timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 --no-clocks | sed "s/^{/{\"lib\": \"$lib\", /" >> gpurun_out/gather_configs.jsonl
  done
done
export KB_OVERLAP=0 KB_REPS=3; bash tools/gpu_var_only.sh
