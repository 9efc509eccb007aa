# full ncu capture of one k_visc_div launch (512^3 weak config via tools/kbench.py)
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
export KB_N=512 KB_REPS=1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_visc_div" -s 3 -c 1 -o gpurun_out/prof_vdiv python tools/kbench.py > gpurun_out/ncu_vdiv.log 2>&1
ncu -i gpurun_out/prof_vdiv.ncu-rep --page raw --csv > gpurun_out/vdiv_raw.csv 2>/dev/null
ncu -i gpurun_out/prof_vdiv.ncu-rep --page source --csv --print-source sass > gpurun_out/vdiv_sass.csv 2>/dev/null
ncu -i gpurun_out/prof_vdiv.ncu-rep --page details > gpurun_out/vdiv_details.txt 2>/dev/null
