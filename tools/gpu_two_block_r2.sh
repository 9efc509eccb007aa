#!/bin/bash
# two 512^3 blocks on one GPU (the per-GPU shape of the N=2 weak run, twice): local copies vs the
# multi-rank exchange code through the NCCL loopback, serial vs overlapped stage
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
: > gpurun_out/r02_two_block.jsonl
for lb in 0 1; do for ov in 0 1; do
  KB_BLOCKS=2,1,1 KB_LOOPBACK=$lb KB_OVERLAP=$ov KB_REPS=2 timeout 900 python tools/kbench.py >> gpurun_out/r02_two_block.jsonl 2>> gpurun_out/r02_two_block.err
done; done
