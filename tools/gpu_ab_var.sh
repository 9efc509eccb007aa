#!/bin/bash
# bitwise A/B hashes (tools/abhash.py) + kbench timing of build/variants/*.so
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
bash tools/gpu_ab.sh
VAR_OUT=${VAR_OUT:-variants_ab} bash tools/gpu_var_r2.sh
cat gpurun_out/ab.jsonl; cut -c1-330 gpurun_out/${VAR_OUT:-variants_ab}.jsonl
