# Pass-1 / pass-2 construct time of huge regions (run under gpurun).
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
for g in ${GS_MIN:-128}; do
  for n in ${PROBE_SIZES:-700 1000 1500 2000 3000}; do
    ACO_GS_MIN_THREADS=$g PROBE_N=$n timeout 300 python tools/size_probe.py 2>&1 | sed "s/^/gs_min $g: /"
  done
done | tee gpurun_out/probe.log
