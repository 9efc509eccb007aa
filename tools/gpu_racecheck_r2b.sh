#!/bin/bash
# racecheck of the late round-2 kernels (xi column-major ring, zeta ring U_in, k_visc_exp_tiled);
# the 100-step RK3 tests are left out (the racecheck process dies on long runs, no hazard reported)
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
SEL="rhs_parity_terms or rhs_parity_sod or decomposition_invariance or overlapped_stage or rhs_parity_expanded or second_metrics or expanded_constant_mu or rk3_parity_expanded"
timeout 2400 compute-sanitizer --tool racecheck --target-processes all --print-limit 20 \
   python -m pytest tests/test_gpu_parity.py tests/test_gpu_metrics27.py -q -x -k "$SEL" > gpurun_out/racecheck_r2b.log 2>&1
echo "exit $?" >> gpurun_out/racecheck_r2b.log
