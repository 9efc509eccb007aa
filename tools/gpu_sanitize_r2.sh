#!/bin/bash
# round 2: compute-sanitizer (all four tools) on the changed sweeps (ring layout, prefetch slots,
# cubic approximations), the NCCL loopback path, the overlapped stage and the sibling AMR kernels
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
SEL="rhs_parity_terms or decomposition or overlapped or loopback or abutting or disjoint or graph_dropped or non_finite"
for tool in memcheck racecheck initcheck synccheck; do
  timeout 2400 compute-sanitizer --tool $tool --target-processes all --print-limit 20 \
     python -m pytest tests/test_gpu_amr.py tests/test_gpu_parity.py -q -x -k "$SEL" > gpurun_out/sanitize_r2_$tool.log 2>&1
  echo "exit $?" >> gpurun_out/sanitize_r2_$tool.log
done
