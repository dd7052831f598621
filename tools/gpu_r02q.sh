# r02q: compile-switch A/B (lean launch bound -> register budget; scan4 word prefetch)
set -x
O=gpurun_out/r02q; mkdir -p $O
B="python bench.py --steps 3 --warmup 3 --parity off --no-cpu-baseline --e2e-steps 1"
for v in main lb256 lb384 pf main; do
  if [ $v = main ]; then unset ACO_LIB_VARIANT; else export ACO_LIB_VARIANT=$v; fi
  timeout 900 $B > $O/c3_$v.json 2>$O/c3_$v.err
  mv $O/c3_$v.json $O/c3_${v}_$(date +%s).json
done
unset ACO_LIB_VARIANT
for v in lb256 pf; do ACO_LIB_VARIANT=$v MB_SIZES=200,450 timeout 900 python tools/microbench.py > $O/mb_$v.txt 2>&1; done
MB_SIZES=200,450 timeout 900 python tools/microbench.py > $O/mb_main.txt 2>&1
for f in $O/*.json; do echo -n "$f "; python -c "import json,sys; d=json.load(open('$f')); print(d['ms_per_step'], d['phase_ms_per_step']['construct'])"; done
tail -n 2 $O/mb_*.txt
