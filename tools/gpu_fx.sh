# FP64-count variant: kernel times + parity subset with the variant lib (round 2)
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
VAR_OUT=fx_var bash tools/gpu_var_r2.sh
CROCCO_LIB=$PWD/build/variants/libcrocco_fx.so timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "not native_library_loaded" > gpurun_out/fx_parity.log 2>&1; echo "exit $?" >> gpurun_out/fx_parity.log
