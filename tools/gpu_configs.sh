# all BASELINE configs on one GPU (bench.py --config), plus the default bench line
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
: > gpurun_out/configs.jsonl
for c in sod vortex tgv ramp dmr weak; do
  timeout 900 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 >> gpurun_out/configs.jsonl 2>> gpurun_out/configs.err
done
