python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
timeout 900 python -m pytest tests -x -q -m gpu --timeout 150 2>&1 | tail -3
for e in ACO_RECORD_MB=0 ACO_RECORD_MB=100000; do
  for w in ${WL:-c1 c2 c4 c3 c5}; do
    echo "== $e $w: $(env $e timeout 400 python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | cut -c1-400 | grep -o '"ms_per_step": [0-9.]*\|"phase_ms_per_step": {[^}]*}' | tr '\n' ' ')"
  done
done
