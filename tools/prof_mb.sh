# ncu capture (full set + source) of the construct launches of the per-size
# microbenchmark at one size (run under gpurun): MB_N (default 450).
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
MB_SIZES=${MB_N:-450} MB_ITERS=1 MB_MIN_REGIONS=${MB_REG:-160} timeout 900 ncu --set full --clock-control none --import-source on \
  --kernel-name-base demangled -k regex:"${KRE:-k_construct}" -s ${SKIP:-0} -c ${PROF_COUNT:-1} -o gpurun_out/prof_mb python tools/microbench.py > gpurun_out/prof_mb.log 2>&1
ncu -i gpurun_out/prof_mb.ncu-rep --page raw --csv > gpurun_out/prof_mb_raw.csv 2>&1
ncu -i gpurun_out/prof_mb.ncu-rep --page source --csv --print-source cuda,sass > gpurun_out/prof_mb_src.csv 2>&1
ls -la gpurun_out
