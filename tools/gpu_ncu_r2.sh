# round 2: ncu --set full of the three sweeps + viscous kernel at 512^3 (kbench workload, one stage each)
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
TAG=${NCU_TAG:-r02}
KB_REPS=1 KB_OVERLAP=0 timeout 1200 ncu --set full --import-source on --clock-control none \
  -k regex:"k_sweep_s|k_visc_tiled" -s 4 -c 4 -o gpurun_out/${TAG}_kernels -f python tools/kbench.py > gpurun_out/${TAG}_ncu.log 2>&1
echo "ncu exit $?" >> gpurun_out/${TAG}_ncu.log
