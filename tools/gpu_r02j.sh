# r02j: lazy kill derivation in the lean pass-2 layout (A/B + parity with it on)
set -x
O=gpurun_out/r02j; mkdir -p $O
ACO_LAZY_KILLS=1 timeout 1500 python -m pytest tests -q -x -m gpu -p no:cacheprovider > $O/gpu_tests_lazy.log 2>&1; echo "pytest exit $?" >> $O/gpu_tests_lazy.log
B="python bench.py --steps 3 --warmup 3 --parity off --no-cpu-baseline --e2e-steps 1"
for r in 1 2; do
  ACO_LAZY_KILLS=0 timeout 900 $B > $O/c3_lazy0_$r.json 2>$O/c3_lazy0_$r.err
  ACO_LAZY_KILLS=1 timeout 900 $B > $O/c3_lazy1_$r.json 2>$O/c3_lazy1_$r.err
done
ACO_LAZY_KILLS=1 timeout 900 $B --workload c5 > $O/c5_lazy1.json 2>$O/c5_lazy1.err
ACO_LAZY_KILLS=0 timeout 900 $B --workload c5 > $O/c5_lazy0.json 2>$O/c5_lazy0.err
ACO_LAZY_KILLS=0 MB_SIZES=200,450 timeout 900 python tools/microbench.py > $O/mb_lazy0.txt 2>&1
ACO_LAZY_KILLS=1 MB_SIZES=200,450 timeout 900 python tools/microbench.py > $O/mb_lazy1.txt 2>&1
tail -3 $O/gpu_tests_lazy.log
for f in $O/*.json; do echo -n "$f "; python -c "import json,sys; d=json.load(open('$f')); print(d['ms_per_step'], d['phase_ms_per_step']['construct'])"; done
cat $O/mb_lazy0.txt $O/mb_lazy1.txt
