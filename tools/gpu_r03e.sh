# A/B: huge regions with the per-ant state in shared memory, exact reservation
# (L1 keeps the rest), one or several waves, 64 / 128 register bound.
set -x
O=gpurun_out/r03e; mkdir -p $O
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py huge1 ACO_HUGE_MINB=1 > /dev/null
b() {  # name, env...
  name=$1; shift
  for w in ${WL:-c4 c5}; do
    r=$(env "$@" timeout 600 python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline --parity off 2>$O/$name.$w.err | tail -1)
    echo "== $name $w: $(echo "$r" | grep -o '"ms_per_step": [0-9.]*\|"phase_ms_per_step": {[^}]*}' | tr '\n' ' ')" | tee -a $O/ab.log
  done
}
b default ACO_X=0
b huge_exact ACO_HUGE_SMEM=1
b huge_old ACO_HUGE_SMEM=1 ACO_HUGE_EXACT=0
b huge1_w ACO_LIB_VARIANT=huge1 ACO_HUGE_SMEM=1 ACO_HUGE_K=1 ACO_HUGE_WAVES=1
b huge1_w_l8 ACO_LIB_VARIANT=huge1 ACO_HUGE_SMEM=1 ACO_HUGE_K=1 ACO_HUGE_WAVES=1 ACO_GS_LANES=8,8
b huge2_w96 ACO_HUGE_SMEM=1 ACO_HUGE_WAVES=1 ACO_HUGE_SMEM_KB=96
cat $O/ab.log
