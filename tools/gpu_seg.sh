#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
: > gpurun_out/seg.jsonl
for lib in s32 s16 s8; do
  for c in vortex tgv sod; do
    CROCCO_LIB=$PWD/build/variants/libcrocco_$lib.so timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 --no-clocks | sed "s/^{/{\"lib\": \"$lib\", /" >> gpurun_out/seg.jsonl
  done
done
