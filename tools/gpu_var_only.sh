cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
: > gpurun_out/variants.jsonl
for r in 1 2; do
for v in build/variants/libcrocco_*.so; do
  CROCCO_LIB=$PWD/$v timeout 300 python tools/kbench.py >> gpurun_out/variants.jsonl 2>> gpurun_out/variants.err
done
done
