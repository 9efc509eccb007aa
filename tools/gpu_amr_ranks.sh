#!/bin/bash
# inter-level AMR boxes (crocco_amr_plan): every GPU AMR test, then memcheck of the loopback path
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_amr.py -q -x > gpurun_out/amr_ranks_tests.log 2>&1
echo "pytest exit $?" >> gpurun_out/amr_ranks_tests.log
timeout 1200 compute-sanitizer --tool memcheck --target-processes all python -m pytest tests/test_gpu_amr.py -q -x \
  -k "loopback or two_level_rk3 or average_down" > gpurun_out/amr_ranks_memcheck.log 2>&1
echo "exit $?" >> gpurun_out/amr_ranks_memcheck.log
