#!/bin/bash
# round 2: cost of the multi-rank exchange code on one GPU (NCCL loopback), serial vs overlapped stage
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
: > gpurun_out/loopback_r2.jsonl
for cfg in "0 0" "0 1" "1 0" "1 1"; do set -- $cfg
  KB_LOOPBACK=$1 KB_OVERLAP=$2 timeout 600 python tools/kbench.py >> gpurun_out/loopback_r2.jsonl 2>> gpurun_out/loopback_r2.err
done
