#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
SEL="rhs_parity_terms or decomposition_invariance or overlapped_stage or full_size_config_sampled and (weak or ramp)"
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "$SEL" > gpurun_out/vk_tests.log 2>&1; echo "exit $?" >> gpurun_out/vk_tests.log
export KB_OVERLAP=0 KB_REPS=3; bash tools/gpu_var_only.sh
