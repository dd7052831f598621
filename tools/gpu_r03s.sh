# A/B: regions above ACO_HUGE_MIN_N on the huge-region kernels (C5's n = 1,000 row; C5 sweep rows).
set -x
O=gpurun_out/r03s; mkdir -p $O
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
ACO_HUGE_MIN_N=600 ACO_SYNC_DEBUG=1 timeout 600 python -m pytest tests/test_gpu_coverage.py -q -k "huge" -p no:cacheprovider > $O/t.log 2>&1; tail -2 $O/t.log
b() {  # name workload env...
  name=$1; w=$2; shift 2
  r=$(env "$@" timeout 600 python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline --parity off 2>$O/$name.$w.err | tail -1)
  echo "== $name $w: $(echo "$r" | grep -o '"ms_per_step": [0-9.]*\|"phase_ms_per_step": {[^}]*}' | tr '\n' ' ')" | tee -a $O/ab.log
}
b default c5 ACO_X=0
b min600 c5 ACO_HUGE_MIN_N=600
b min800 c5 ACO_HUGE_MIN_N=800
b min400 c5 ACO_HUGE_MIN_N=400
timeout 900 python tools/c5_sweep.py --sizes 500,1000 > $O/sweep_default.md 2>/dev/null
ACO_HUGE_MIN_N=400 timeout 900 python tools/c5_sweep.py --sizes 500,1000 > $O/sweep_400.md 2>/dev/null
cat $O/ab.log; cat $O/sweep_default.md $O/sweep_400.md | grep "^| [0-9]"
