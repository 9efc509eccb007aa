#!/bin/bash
# XDIV variants (xi viscous divergence fused into k_visc_tiled): parity subset per variant, then timing
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
SEL="rhs_parity_terms or decomposition_invariance or rk3_100_steps or free_stream or rhs_parity_sutherland or rhs_minimum_block or ramp_downscaled or full_size_config_sampled and weak"
: > gpurun_out/xdiv_tests.log
for v in x16 x24 x32; do
  echo "== $v" >> gpurun_out/xdiv_tests.log
  CROCCO_LIB=$PWD/build/variants/libcrocco_$v.so timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "$SEL" >> gpurun_out/xdiv_tests.log 2>&1
  echo "exit $?" >> gpurun_out/xdiv_tests.log
done
export KB_OVERLAP=0 KB_REPS=3
bash tools/gpu_var_only.sh
