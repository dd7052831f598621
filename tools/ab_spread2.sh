python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
for e in "ACO_SPREAD=0" "ACO_SPREAD=1 ACO_SPREAD_LANES=1 ACO_SPREAD_CAP=32" "ACO_SPREAD=1 ACO_SPREAD_LANES=1 ACO_SPREAD_CAP=64" "ACO_SPREAD=1 ACO_SPREAD_LANES=2 ACO_SPREAD_CAP=32" "ACO_SPREAD=1 ACO_SPREAD_LANES=4 ACO_SPREAD_CAP=16" "ACO_SPREAD=1 ACO_SPREAD_LANES=1 ACO_SPREAD_CAP=128"; do
  for w in c2 c1; do
    echo "== $e $w: $(env $e timeout 300 python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | grep -o '"ms_per_step": [0-9.]*\|"phase_ms_per_step": {[^}]*}' | tr '\n' ' ')"
  done
done
