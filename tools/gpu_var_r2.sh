# round 2: time build/variants/*.so with tools/kbench.py (512^3 bench workload, per-kernel CUDA events)
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
OUT=gpurun_out/${VAR_OUT:-variants_r2}.jsonl
: > $OUT
export KB_OVERLAP=0
for r in ${VAR_REPS:-1 2}; do
for v in build/variants/libcrocco_*.so; do
  CROCCO_LIB=$PWD/$v timeout 300 python tools/kbench.py >> $OUT 2>> gpurun_out/variants.err
done
done
if [ -n "$VAR_CHECK" ]; then
  for v in $VAR_CHECK; do
    CROCCO_LIB=$PWD/build/variants/libcrocco_$v.so timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "rhs_parity_terms or decomposition or viscous_parity" > gpurun_out/varcheck_$v.log 2>&1
    echo "$v pytest exit $?" >> gpurun_out/varcheck_$v.log
  done
fi
