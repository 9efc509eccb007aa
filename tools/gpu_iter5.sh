# correctness + limiter on/off timing
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x --durations=8 ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1
echo "pytest exit $?" >> gpurun_out/pytest_gpu.log
export KB_OVERLAP=0
: > gpurun_out/variants.jsonl
for lim in 0 1 3; do KB_LIM=$lim timeout 300 python tools/kbench.py >> gpurun_out/variants.jsonl 2>> gpurun_out/variants.err; done
