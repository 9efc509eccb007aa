#!/bin/bash
# NEXT-3 27-component metrics / expanded viscous form: GPU parity + stage timing vs the default form
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_metrics27.py -q -x > gpurun_out/pytest_m27.log 2>&1
echo "pytest m27 exit $?" >> gpurun_out/pytest_m27.log
: > gpurun_out/kb_m27.jsonl
for vf in 0 1; do KB_N=512 KB_REPS=2 KB_OVERLAP=0 KB_VISC_FORM=$vf timeout 600 python tools/kbench.py >> gpurun_out/kb_m27.jsonl 2>> gpurun_out/kb_m27.err; done
