python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
for e in "ACO_FEW_WIDE=0" "ACO_FEW_WIDE=1" "ACO_FEW_WIDE=1 ACO_SPREAD=1 ACO_SPREAD_LANES=1 ACO_SPREAD_CAP=64"; do
  for w in c2 c1; do
    echo "== $e $w: $(env $e timeout 300 python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | grep -o '"ms_per_step": [0-9.]*\|"phase_ms_per_step": {[^}]*}' | tr '\n' ' ')"
  done
done
timeout 900 python -m pytest tests -x -q -m gpu --timeout 150 2>&1 | tail -3
