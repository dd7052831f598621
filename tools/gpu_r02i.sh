# r02i: GPU tests on the sparse ready-time slots; A/B slots (C3, C5, C2), C4 with pass-1 GS wide
set -x
O=gpurun_out/r02i; mkdir -p $O
timeout 1500 python -m pytest tests -q -x -m gpu -p no:cacheprovider > $O/gpu_tests.log 2>&1; echo "pytest exit $?" >> $O/gpu_tests.log
B="python bench.py --steps 3 --warmup 3 --parity off --no-cpu-baseline --e2e-steps 1"
for w in c3 c5 c2; do
  ACO_SLOTS=0 timeout 900 $B --workload $w > $O/${w}_slots0.json 2>$O/${w}_slots0.err
  timeout 900 $B --workload $w > $O/${w}_slots1.json 2>$O/${w}_slots1.err
done
timeout 900 $B --workload c4 > $O/c4.json 2>$O/c4.err
timeout 600 $B --workload c1 > $O/c1.json 2>$O/c1.err
MB_SIZES=200,450 timeout 900 python tools/microbench.py > $O/mb_slots1.txt 2>&1
ACO_SLOTS=0 MB_SIZES=200,450 timeout 900 python tools/microbench.py > $O/mb_slots0.txt 2>&1
tail -3 $O/gpu_tests.log
for f in $O/*.json; do echo -n "$f "; python -c "import json,sys; d=json.load(open('$f')); print(d['ms_per_step'], d['phase_ms_per_step']['construct'])"; done
cat $O/mb_slots0.txt $O/mb_slots1.txt
