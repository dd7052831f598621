# A/B: ACO_HUGE_MIN_N on config 3 (regions up to n = 500) and config 4.
set -x
O=gpurun_out/r03t; mkdir -p $O
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
b() {  # name workload env...
  name=$1; w=$2; shift 2
  r=$(env "$@" timeout 600 python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline --parity off 2>$O/$name.$w.err | tail -1)
  echo "== $name $w: $(echo "$r" | grep -o '"ms_per_step": [0-9.]*\|"phase_ms_per_step": {[^}]*}' | tr '\n' ' ')" | tee -a $O/ab.log
}
b default c3 ACO_X=0
b min400 c3 ACO_HUGE_MIN_N=400
b min300 c3 ACO_HUGE_MIN_N=300
b min200 c3 ACO_HUGE_MIN_N=200
b min300 c5 ACO_HUGE_MIN_N=300
b min200 c5 ACO_HUGE_MIN_N=200
cat $O/ab.log
