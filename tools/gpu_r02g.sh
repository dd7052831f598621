# r02g: GPU tests, A/B lean pass-1 layout (C3, C5), fill rule, fused coins (C1)
set -x
O=gpurun_out/r02g; mkdir -p $O
timeout 1500 python -m pytest tests -q -x -m gpu -p no:cacheprovider > $O/gpu_tests.log 2>&1; echo "pytest exit $?" >> $O/gpu_tests.log
B="python bench.py --steps 3 --warmup 3 --parity off --no-cpu-baseline --e2e-steps 1"
for w in c3 c5; do
  ACO_LEAN1=0 timeout 900 $B --workload $w > $O/${w}_lean0.json 2>$O/${w}_lean0.err
  timeout 900 $B --workload $w > $O/${w}_lean1.json 2>$O/${w}_lean1.err
done
ACO_LEAN1_GAIN=0 timeout 900 $B --workload c3 > $O/c3_lean1_g0.json 2>$O/c3_lean1_g0.err
ACO_LEAN1_GAIN=50 timeout 900 $B --workload c3 > $O/c3_lean1_g50.json 2>$O/c3_lean1_g50.err
for w in c1 c2; do timeout 600 $B --workload $w > $O/${w}.json 2>$O/${w}.err; done
MB_SIZES=200,450,900 timeout 900 python tools/microbench.py > $O/mb_lean1.txt 2>&1
ACO_LEAN1=0 MB_SIZES=200,450,900 timeout 900 python tools/microbench.py > $O/mb_lean0.txt 2>&1
tail -3 $O/gpu_tests.log
for f in $O/*.json; do echo -n "$f "; python -c "import json,sys; d=json.load(open('$f')); print(d['ms_per_step'], d['phase_ms_per_step']['construct'], d['gpu_launches'])"; done
cat $O/mb_lean0.txt $O/mb_lean1.txt
