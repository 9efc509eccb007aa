# correctness + overlap on/off timing + default bench line
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x --durations=5 ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1
echo "pytest exit $?" >> gpurun_out/pytest_gpu.log
: > gpurun_out/variants.jsonl
for ov in 0 1; do KB_OVERLAP=$ov timeout 300 python tools/kbench.py >> gpurun_out/variants.jsonl 2>> gpurun_out/variants.err; done
timeout 900 python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/bench.log 2>&1
echo "bench exit $?" >> gpurun_out/bench.log
