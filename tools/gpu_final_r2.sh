#!/bin/bash
# round 2 (late): full GPU suite + smoke on HEAD, then every bench config once
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02g_smoke.log 2>&1; echo "smoke exit $?" >> gpurun_out/r02g_smoke.log
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/r02g_gputest.log 2>&1; echo "pytest exit $?" >> gpurun_out/r02g_gputest.log
bash tools/gpu_configs_r2.sh
