#!/bin/bash
# compute-sanitizer on the fused xi viscous divergence (k_visc_tiled with XDIV) incl. the overlapped stage
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
SEL="rhs_parity_terms or rhs_parity_sutherland or decomposition_invariance or overlapped_stage or rhs_minimum_block"
for tool in memcheck racecheck initcheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --target-processes all --print-limit 20 \
     python -m pytest tests/test_gpu_parity.py -q -x -k "$SEL" > gpurun_out/sanitize_xdiv_$tool.log 2>&1
  echo "exit $?" >> gpurun_out/sanitize_xdiv_$tool.log
done
