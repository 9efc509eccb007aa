#!/bin/bash
# end of round 2: evidence on HEAD (GPU suite, smoke, bench, reference arm, ncu launch list), then
# compute-sanitizer memcheck + racecheck on the sweeps' predicated copies / branch-free flux
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
TAG=r02n bash tools/gpu_evidence_r2.sh
SEL="rhs_parity_terms or decomposition or overlapped or rhs_parity_sod or minimum_block"
for tool in memcheck racecheck; do
  timeout 1500 compute-sanitizer --tool $tool --target-processes all --print-limit 20 \
     python -m pytest tests/test_gpu_parity.py -q -x -k "$SEL" > gpurun_out/r02n_sanitize_$tool.log 2>&1
  echo "exit $?" >> gpurun_out/r02n_sanitize_$tool.log
done
