python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
timeout 900 python -m pytest tests -x -q -m gpu --timeout 150 2>&1 | tail -3
for e in ACO_PIPELINE=0 ACO_PIPELINE=1; do
  for w in ${WL:-c3 c5 c2}; do
    echo "== $e $w: $(env $e timeout 400 python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | grep -o '"ms_per_step": [0-9.]*\|"phase_ms_per_step": {[^}]*}\|"gpu_launches": [0-9]*' | tr '\n' ' ')"
  done
done
