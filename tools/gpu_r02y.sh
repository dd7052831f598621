# r02y: classes reserve only the shared memory they need (the rest becomes L1)
set -x
O=gpurun_out/r02y; mkdir -p $O
B="python bench.py --steps 3 --warmup 3 --parity off --no-cpu-baseline --e2e-steps 1"
for v in 1 0 1 0; do ACO_SMEM_EXACT=$v timeout 900 $B > $O/c3_$v.json 2>$O/c3.err; mv $O/c3_$v.json $O/c3_${v}_$(date +%s%N).json; done
for w in c5 c2 c4; do for v in 0 1; do ACO_SMEM_EXACT=$v timeout 900 $B --workload $w > $O/${w}_$v.json 2>$O/$w.err; done; done
ACO_SMEM_EXACT=0 MB_SIZES=60,200,450 timeout 900 python tools/microbench.py > $O/mb_0.txt 2>&1
ACO_SMEM_EXACT=1 MB_SIZES=60,200,450 timeout 900 python tools/microbench.py > $O/mb_1.txt 2>&1
timeout 1500 python -m pytest tests -q -x -m gpu -p no:cacheprovider > $O/gpu_tests.log 2>&1; echo "pytest exit $?" >> $O/gpu_tests.log
tail -2 $O/gpu_tests.log
for f in $O/*.json; do echo -n "$f "; python -c "import json,sys; d=json.load(open('$f')); print(d['ms_per_step'], d['phase_ms_per_step']['construct'])"; done
tail -n 3 $O/mb_*.txt
