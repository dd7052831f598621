# r02t: pass-2 wide/lean size threshold (runtime ACO_WIDE_N)
set -x
O=gpurun_out/r02t; mkdir -p $O
B="python bench.py --steps 3 --warmup 3 --parity off --no-cpu-baseline --e2e-steps 1"
for t in 160,160 160,120 160,104 160,136 160,120; do ACO_WIDE_N=$t timeout 900 $B > $O/c3_$t.json 2>$O/c3_$t.err; mv $O/c3_$t.json $O/c3_${t/,/_}_$(date +%s%N).json; done
for t in 160,160 160,120; do ACO_WIDE_N=$t timeout 900 $B --workload c5 > $O/c5_${t/,/_}.json 2>$O/c5.err; done
ACO_WIDE_N=160,160 MB_SIZES=104,112,120 timeout 900 python tools/microbench.py > $O/mb_160.txt 2>&1
ACO_WIDE_N=104,104 MB_SIZES=104,112,120 timeout 900 python tools/microbench.py > $O/mb_104.txt 2>&1
timeout 1500 python -m pytest tests -q -x -m gpu -p no:cacheprovider > $O/gpu_tests.log 2>&1; echo "pytest exit $?" >> $O/gpu_tests.log
tail -2 $O/gpu_tests.log
for f in $O/*.json; do echo -n "$f "; python -c "import json,sys; d=json.load(open('$f')); print(d['ms_per_step'], d['phase_ms_per_step']['construct'])"; done
tail -n 3 $O/mb_*.txt
