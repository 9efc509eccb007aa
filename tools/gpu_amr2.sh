#!/bin/bash
# AMR tests (incl. the ramp/wall two-level case) + smoke with the two-level step
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1
echo "smoke exit $?" >> gpurun_out/smoke.log
timeout 600 python -m pytest tests/test_gpu_amr.py -q -x > gpurun_out/pytest_amr.log 2>&1
echo "pytest amr exit $?" >> gpurun_out/pytest_amr.log
