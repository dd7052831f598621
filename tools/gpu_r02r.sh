# r02r: lean launch bound 384 (main) + A/B 1-wide variants' register budget (nmb1)
set -x
O=gpurun_out/r02r; mkdir -p $O
timeout 1500 python -m pytest tests -q -x -m gpu -p no:cacheprovider > $O/gpu_tests.log 2>&1; echo "pytest exit $?" >> $O/gpu_tests.log
B="python bench.py --steps 3 --warmup 3 --parity off --no-cpu-baseline --e2e-steps 1"
for r in 1 2; do
  timeout 900 $B > $O/c3_main_$r.json 2>$O/c3_main_$r.err
  ACO_LIB_VARIANT=nmb1 timeout 900 $B > $O/c3_nmb1_$r.json 2>$O/c3_nmb1_$r.err
done
for w in c4 c5 c2; do timeout 900 $B --workload $w > $O/${w}.json 2>$O/${w}.err; done
MB_SIZES=30,60,120,200,450 timeout 900 python tools/microbench.py > $O/mb_main.txt 2>&1
ACO_LIB_VARIANT=nmb1 MB_SIZES=30,60,120 timeout 900 python tools/microbench.py > $O/mb_nmb1.txt 2>&1
tail -3 $O/gpu_tests.log
for f in $O/*.json; do echo -n "$f "; python -c "import json,sys; d=json.load(open('$f')); print(d['ms_per_step'], d['phase_ms_per_step']['construct'])"; done
cat $O/mb_main.txt $O/mb_nmb1.txt
