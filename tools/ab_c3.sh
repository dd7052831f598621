python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
timeout 900 python -m pytest tests -x -q -m gpu --timeout 150 2>&1 | tail -3
for w in ${WL:-c3 c2 c1}; do
  echo "== $w: $(timeout 400 python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | grep -o '"ms_per_step": [0-9.]*\|"phase_ms_per_step": {[^}]*}' | tr '\n' ' ')"
done
