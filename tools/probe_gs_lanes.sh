python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
for l in ${GS_LANES:-4,4 8,8}; do
  for n in ${PROBE_SIZES:-1200 2000 3000}; do
    ACO_GS_LANES=$l PROBE_N=$n timeout 300 python tools/size_probe.py 2>&1 | sed "s/^/gs_lanes $l: /"
  done
done | tee gpurun_out/probe.log
