cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
: > gpurun_out/ab.jsonl
for v in build/variants/libcrocco_*.so; do
  for cfg in "128 2,1,1 0" "144 2,1,2 1" "64 1,1,1 0"; do set -- $cfg
    AB_N=$1 AB_NB=$2 AB_OVERLAP=$3 CROCCO_LIB=$PWD/$v timeout 300 python tools/abhash.py >> gpurun_out/ab.jsonl 2>> gpurun_out/ab.err
  done
done
