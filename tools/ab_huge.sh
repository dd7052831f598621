python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
for e in ACO_IMG_HUGE=0 ACO_IMG_HUGE=1 "ACO_IMG_HUGE=1 ACO_MAX_LANES_HUGE=4,4"; do
  for w in ${WL:-c4 c5}; do
    echo "== $e $w: $(env $e timeout 400 python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | grep -o '"ms_per_step": [0-9.]*\|"phase_ms_per_step": {[^}]*}' | tr '\n' ' ')"
  done
done
