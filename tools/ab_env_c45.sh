# C4 and C5 bench lines per env setting: AB_ENVS="VAR=a VAR=b ..." ("-" = none)
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
for e in ${AB_ENVS:--}; do
  if [ "$e" = "-" ]; then e2=""; else e2="$e"; fi
  for w in c4 c5; do
    echo "== $e $w: $(env $e2 timeout 400 python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | grep -o '"ms_per_step": [0-9.]*' | head -1)"
  done
done
