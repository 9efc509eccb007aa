#!/bin/bash
# AMR row (NEXT-4): GPU parity tests of the two-level path, then the whole GPU suite
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_amr.py -q -x > gpurun_out/pytest_amr.log 2>&1
echo "pytest amr exit $?" >> gpurun_out/pytest_amr.log
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1
echo "pytest exit $?" >> gpurun_out/pytest_gpu.log
