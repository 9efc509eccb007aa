# correctness (default .so) + variant timings + inviscid-only timing of the default
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x --durations=5 ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1
echo "pytest exit $?" >> gpurun_out/pytest_gpu.log
: > gpurun_out/variants.jsonl
for v in build/variants/libcrocco_*.so; do
  CROCCO_LIB=$PWD/$v timeout 300 python tools/kbench.py >> gpurun_out/variants.jsonl 2>> gpurun_out/variants.err
done
KB_TERMS=1 timeout 300 python tools/kbench.py >> gpurun_out/variants.jsonl 2>> gpurun_out/variants.err
