#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
SEL="rhs_parity_terms or decomposition_invariance or rk3_100_steps or rhs_parity_sutherland or rhs_minimum_block or ramp_downscaled or overlapped_stage or full_size_config_sampled and weak"
CROCCO_LIB=$PWD/build/variants/libcrocco_shfl.so timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "$SEL" > gpurun_out/xshfl_tests.log 2>&1
echo "exit $?" >> gpurun_out/xshfl_tests.log
export KB_OVERLAP=0 KB_REPS=3; bash tools/gpu_var_only.sh
