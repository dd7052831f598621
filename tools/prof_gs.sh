# ncu capture of the huge-region (global-state) construct kernels (run under gpurun).
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
PROBE_N=${PROBE_N:-2000} PROBE_ITERS=1 timeout 900 ncu --set full --clock-control none --import-source on \
  --kernel-name-base demangled -k regex:k_construct -c ${PROF_COUNT:-2} -o gpurun_out/prof_gs python tools/size_probe.py > gpurun_out/prof_gs.log 2>&1
ncu -i gpurun_out/prof_gs.ncu-rep --page raw --csv > gpurun_out/prof_gs_raw.csv 2>&1
