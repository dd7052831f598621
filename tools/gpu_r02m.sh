# r02m: u16x2 guard-bit class tests (no byte-SIMD emulation) + pass-1 spread lanes
set -x
O=gpurun_out/r02m; mkdir -p $O
timeout 1500 python -m pytest tests -q -x -m gpu -p no:cacheprovider > $O/gpu_tests.log 2>&1; echo "pytest exit $?" >> $O/gpu_tests.log
B="python bench.py --steps 3 --warmup 3 --parity off --no-cpu-baseline --e2e-steps 1"
for r in 1 2; do timeout 900 $B > $O/c3_$r.json 2>$O/c3_$r.err; done
timeout 900 $B --workload c4 > $O/c4.json 2>$O/c4.err
timeout 900 $B --workload c5 > $O/c5.json 2>$O/c5.err
ACO_FILL_LANES=1,0 timeout 900 $B --workload c5 > $O/c5_fl1.json 2>$O/c5_fl1.err
timeout 900 $B --workload c2 > $O/c2.json 2>$O/c2.err
timeout 900 $B --workload c3 --machine dual > $O/c3_dual.json 2>$O/c3_dual.err
MB_SIZES=200,450 timeout 900 python tools/microbench.py > $O/mb.txt 2>&1
tail -3 $O/gpu_tests.log
for f in $O/*.json; do echo -n "$f "; python -c "import json,sys; d=json.load(open('$f')); print(d['ms_per_step'], d['phase_ms_per_step']['construct'])"; done
cat $O/mb.txt
