#!/bin/bash
# compute-sanitizer on the session-3 kernels: AMR (k_cf_interp, k_average_down), the 27-component
# metrics / expanded viscous form (k_metric2, k_prims4, k_visc_exp), k_check_state
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
SEL="fill_patch_two_levels or average_down or two_level_rk3 or three_level_hierarchy or second_metrics or rhs_parity_expanded or check_state"
for tool in memcheck racecheck initcheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --target-processes all --print-limit 20 \
     python -m pytest tests/test_gpu_amr.py tests/test_gpu_metrics27.py tests/test_gpu_parity.py -q -x -k "$SEL" > gpurun_out/sanitize_s3_$tool.log 2>&1
  echo "exit $?" >> gpurun_out/sanitize_s3_$tool.log
done
