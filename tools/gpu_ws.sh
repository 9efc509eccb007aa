# warp-specialised sweeps: bitwise A/B vs k_sweep_s, kernel times, parity subset (round 2)
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
: > gpurun_out/ws_ab.jsonl
for v in build/variants/libcrocco_*.so; do
  for cfg in "128 2,1,1 0" "144 2,1,2 1" "64 1,1,1 0" "40 1,1,1 0"; do set -- $cfg
    AB_N=$1 AB_NB=$2 AB_OVERLAP=$3 CROCCO_LIB=$PWD/$v timeout 120 python tools/abhash.py >> gpurun_out/ws_ab.jsonl 2>> gpurun_out/ws_ab.err
  done
done
VAR_OUT=ws_var bash tools/gpu_var_r2.sh
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/ws_parity.log 2>&1; echo "exit $?" >> gpurun_out/ws_parity.log
