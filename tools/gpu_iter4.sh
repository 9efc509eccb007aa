# viscous variants (overlap off) + full ncu of the default kernels (overlap off: whole viscous launch)
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
export KB_OVERLAP=0
: > gpurun_out/variants.jsonl
for v in build/variants/libcrocco_*.so; do
  CROCCO_LIB=$PWD/$v timeout 300 python tools/kbench.py >> gpurun_out/variants.jsonl 2>> gpurun_out/variants.err
done
export KB_N=512 KB_REPS=1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"k_sweep|k_visc|k_boxops" -s 7 -c 7 -o gpurun_out/prof_s2 python tools/kbench.py > gpurun_out/ncu_s2.log 2>&1
ncu -i gpurun_out/prof_s2.ncu-rep --page details > gpurun_out/prof_s2_details.txt 2>/dev/null
