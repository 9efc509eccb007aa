# variant timings only (overlap off)
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
export KB_OVERLAP=0
: > gpurun_out/variants.jsonl
for v in build/variants/libcrocco_*.so; do
  CROCCO_LIB=$PWD/$v timeout 300 python tools/kbench.py >> gpurun_out/variants.jsonl 2>> gpurun_out/variants.err
done
