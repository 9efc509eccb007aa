#!/bin/bash
# round 2: tiled expanded viscous kernel (visc_form = 1) vs the global-load version: parity + timing
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
: > gpurun_out/vexp_r2.jsonl
for v in vexp_tiled vexp_old; do
  CROCCO_LIB=$PWD/build/variants/libcrocco_$v.so timeout 900 python -m pytest tests/test_gpu_metrics27.py -q -x > gpurun_out/vexp_$v.log 2>&1
  echo "$v pytest exit $?" >> gpurun_out/vexp_$v.log
  for r in 1 2; do
    CROCCO_LIB=$PWD/build/variants/libcrocco_$v.so KB_OVERLAP=0 KB_VISC_FORM=1 timeout 600 python tools/kbench.py >> gpurun_out/vexp_r2.jsonl 2>> gpurun_out/vexp_r2.err
  done
done
CROCCO_LIB=$PWD/build/variants/libcrocco_vexp_tiled.so compute-sanitizer --tool memcheck python -m pytest tests/test_gpu_metrics27.py -q -x -k "rhs_parity" > gpurun_out/vexp_memcheck.log 2>&1
echo "memcheck exit $?" >> gpurun_out/vexp_memcheck.log
