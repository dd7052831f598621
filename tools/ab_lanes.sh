python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
for lanes in 8,1 8,2 8,4; do
  echo "== ACO_MAX_LANES_WIDE=$lanes"
  ACO_MAX_LANES_WIDE=$lanes MB_SIZES=200,300,450 timeout 400 python tools/microbench.py
done
