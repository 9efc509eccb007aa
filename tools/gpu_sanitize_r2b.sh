#!/bin/bash
# round 2 (late): sanitizers on the xi column-major ring, the zeta ring U_in and k_visc_exp_tiled
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
SEL="rhs_parity_terms or rhs_parity_sod or decomposition_invariance or rk3_100_steps_parity or overlapped_stage"
for tool in memcheck racecheck initcheck synccheck; do
  timeout 2400 compute-sanitizer --tool $tool --target-processes all --print-limit 20 \
     python -m pytest tests/test_gpu_parity.py tests/test_gpu_metrics27.py -q -x -k "$SEL or rhs_parity_expanded or second_metrics" > gpurun_out/sanitize_r2b_$tool.log 2>&1
  echo "exit $?" >> gpurun_out/sanitize_r2b_$tool.log
done
