# Bench lines for every config and SURVEY 8(f) mode (run under gpurun, 1 GPU).
# Each JSON line goes to $BM_OUT/bench_<name>.json (default gpurun_out/).
O=${BM_OUT:-gpurun_out}; mkdir -p $O
run() {  # name, args...
  name=$1; shift
  timeout 900 python bench.py --steps ${BM_STEPS:-5} --warmup 3 "$@" 2>$O/bench_$name.err | tail -1 > $O/bench_$name.json
  echo "== $name: $(cut -c1-160 $O/bench_$name.json)"
}
for w in ${MATRIX:-c3 c1 c2 c4 c5 dual weighted policy mix stall50 rlmin rlmid ref}; do
  case $w in
    c1|c2|c3|c4|c5) run $w --workload $w ;;
    dual) run c3_dual --machine dual ;;
    weighted) run c3_weighted --passes 4 --ws-weight 4 ;;
    policy) run c3_paper_policy --policy paper ;;
    mix) run c3_heur_mix --heur-mix 1 ;;
    rlmin) run c3_rl_min --rl-limit 1 ;;
    rlmid) run c3_rl_mid --rl-limit 2 ;;
    stall50) run c3_stall50 --stall-num 2 ;;
    ref) run c3_reference --impl reference ;;
  esac
done
