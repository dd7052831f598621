# Bulk-copy staging + one-launch finalize: GPU tests, C3 / C2 A/B; huge-region sweep (C4).
set -x
O=gpurun_out/r03f; mkdir -p $O
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py nobulk ACO_BULK_STAGE=0 > /dev/null
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py huge1 ACO_HUGE_MINB=1 > /dev/null
timeout 1500 python -m pytest tests -q -m gpu -x -p no:cacheprovider > $O/gpu_tests.log 2>&1; echo "pytest exit $?" >> $O/gpu_tests.log
tail -5 $O/gpu_tests.log
b() {  # name workload env...
  name=$1; w=$2; shift 2
  r=$(env "$@" timeout 600 python bench.py --workload $w --steps 5 --warmup 3 --no-cpu-baseline --parity off 2>$O/$name.$w.err | tail -1)
  echo "== $name $w: $(echo "$r" | grep -o '"ms_per_step": [0-9.]*\|"phase_ms_per_step": {[^}]*}' | tr '\n' ' ')" | tee -a $O/ab.log
}
b bulk c3 ACO_X=0
b nobulk c3 ACO_LIB_VARIANT=nobulk
b bulk c3 ACO_X=0
b nobulk c3 ACO_LIB_VARIANT=nobulk
b bulk c2 ACO_X=0
b nobulk c2 ACO_LIB_VARIANT=nobulk
for cfg in "8,8 1" "8,8 2" "4,4 1" "4,4 2" "4,4 4" "16,8 1" "8,4 2" "8,4 1"; do
  set -- $cfg
  b "huge1_l${1}_k$2" c4 ACO_LIB_VARIANT=huge1 ACO_HUGE_SMEM=1 ACO_HUGE_WAVES=1 ACO_GS_LANES=$1 ACO_HUGE_K=$2
done
cat $O/ab.log
