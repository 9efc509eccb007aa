#!/bin/bash
# round 2: racecheck per test (verbose), NCCL loopback excluded (NCCL's own kernels under racecheck)
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
SEL="(overlapped or graph_dropped or non_finite or decomposition_invariance) and not loopback"
timeout 2400 compute-sanitizer --tool racecheck --target-processes all --print-limit 20 \
   python -m pytest tests/test_gpu_amr.py tests/test_gpu_parity.py -v -x -k "$SEL" > gpurun_out/sanitize_r2_racecheck2.log 2>&1
echo "exit $?" >> gpurun_out/sanitize_r2_racecheck2.log
