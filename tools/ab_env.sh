# A/B of launch-policy environment settings on the C3 bench: AB_ENVS="VAR=a VAR=b ..." (one run each; "-" = none)
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
for e in ${AB_ENVS:--}; do
  echo "== $e"
  if [ "$e" = "-" ]; then e=""; fi
  env $e MB_SIZES=${MB_SIZES:-200,300,450} timeout 400 python tools/microbench.py
  env $e timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | cut -c1-200
done
