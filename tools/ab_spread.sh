python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
timeout 900 python -m pytest tests -x -q -m gpu --timeout 150 2>&1 | tail -3
for e in ACO_SPREAD=0 ACO_SPREAD=1; do
  for w in c2 c1; do
    echo "== $e $w: $(env $e timeout 300 python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | cut -c1-150)"
  done
done
