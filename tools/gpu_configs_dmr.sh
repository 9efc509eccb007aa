cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 900 python bench.py --config dmr --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/dmr.jsonl 2> gpurun_out/dmr.err
timeout 900 python -m pytest tests -m gpu -q -k full_size > gpurun_out/pytest_full.log 2>&1
