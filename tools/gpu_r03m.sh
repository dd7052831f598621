# A/B: huge regions with the image staged in shared memory too (ACO_HUGE_IMG).
set -x
O=gpurun_out/r03m; mkdir -p $O
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
ACO_HUGE_IMG=1 ACO_SYNC_DEBUG=1 timeout 600 python -m pytest tests/test_gpu_coverage.py -q -k "huge or config4" -p no:cacheprovider > $O/huge_tests.log 2>&1; echo "pytest exit $?" >> $O/huge_tests.log
tail -3 $O/huge_tests.log
b() {  # name workload env...
  name=$1; w=$2; shift 2
  r=$(env "$@" timeout 600 python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline --parity off 2>$O/$name.$w.err | tail -1)
  echo "== $name $w: $(echo "$r" | grep -o '"ms_per_step": [0-9.]*\|"phase_ms_per_step": {[^}]*}' | tr '\n' ' ')" | tee -a $O/ab.log
}
b default c4 ACO_X=0
b img_l8 c4 ACO_HUGE_IMG=1
b img_l16 c4 ACO_HUGE_IMG=1 ACO_HUGE_LANES=16,16
b img_l4 c4 ACO_HUGE_IMG=1 ACO_HUGE_LANES=4,4
b img_l16_8 c4 ACO_HUGE_IMG=1 ACO_HUGE_LANES=16,8
b default c5 ACO_X=0
b img_l8 c5 ACO_HUGE_IMG=1
cat $O/ab.log
