# A/B of compile-time variants (built beforehand with build.py <variant> DEFS) on the per-size microbenchmark.
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py
for v in ${AB_VARIANTS:-""}; do
  echo "== variant [$v]"
  ACO_LIB_VARIANT=$v MB_SIZES=${MB_SIZES:-60,120,250,450} timeout 400 python tools/microbench.py
done
