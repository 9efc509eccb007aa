#!/bin/bash
# shorter viscous slabs for small boxes: size sweep + the viscous parity / decomposition / overlap tests
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
python bench.py --config size_sweep --warmup 2 --no-cpu-baseline > gpurun_out/r02_size_sweep_slab.jsonl 2> gpurun_out/size_sweep_slab.err
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_amr.py -q -x -k "viscous or decomposition or overlap or terms or rk3 or two_level" > gpurun_out/slab_small_tests.log 2>&1
echo "pytest exit $?" >> gpurun_out/slab_small_tests.log
for cfg in tgv ramp; do timeout 900 python bench.py --config $cfg --steps 5 --warmup 3 --no-cpu-baseline >> gpurun_out/slab_small_cfgs.jsonl 2>/dev/null; done
