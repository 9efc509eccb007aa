# variant A/B incl. the WENO-limiter path (KB_LIM=1), then the parity file with the variant lib
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
VAR_REPS="1 2 3" VAR_OUT=fx_var bash tools/gpu_var_r2.sh
: > gpurun_out/fx_lim.jsonl
for v in build/variants/libcrocco_*.so; do KB_LIM=1 CROCCO_LIB=$PWD/$v timeout 300 python tools/kbench.py >> gpurun_out/fx_lim.jsonl 2>> gpurun_out/variants.err; done
CROCCO_LIB=$PWD/build/variants/libcrocco_fx.so timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "not native_library_loaded" > gpurun_out/fx_parity.log 2>&1; echo "exit $?" >> gpurun_out/fx_parity.log
