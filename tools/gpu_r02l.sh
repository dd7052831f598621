# r02l: A/B tau-row L1 prefetch (C3, C4, C5), spread lanes for C2
set -x
O=gpurun_out/r02l; mkdir -p $O
B="python bench.py --steps 3 --warmup 3 --parity off --no-cpu-baseline --e2e-steps 1"
for pf in 0 3 1 2; do ACO_TAU_PREFETCH=$pf timeout 900 $B > $O/c3_pf$pf.json 2>$O/c3_pf$pf.err; done
for pf in 0 12 4; do ACO_TAU_PREFETCH=$pf timeout 900 $B --workload c4 > $O/c4_pf$pf.json 2>$O/c4_pf$pf.err; done
for pf in 0 15; do ACO_TAU_PREFETCH=$pf timeout 900 $B --workload c5 > $O/c5_pf$pf.json 2>$O/c5_pf$pf.err; done
for fl in 0,0 2,2 4,4 4,1 1,4; do ACO_FILL_LANES=$fl timeout 900 $B --workload c2 > $O/c2_fl${fl/,/_}.json 2>$O/c2_fl${fl/,/_}.err; done
ACO_TAU_PREFETCH=15 timeout 1500 python -m pytest tests -q -x -m gpu -k "global_state or lean or config3 or config4 or colony" -p no:cacheprovider > $O/gpu_tests_pf.log 2>&1; echo "pytest exit $?" >> $O/gpu_tests_pf.log
ACO_FILL_LANES=4,4 timeout 900 python -m pytest tests -q -x -m gpu -k "config2" -p no:cacheprovider > $O/gpu_tests_fl.log 2>&1; echo "pytest exit $?" >> $O/gpu_tests_fl.log
tail -2 $O/gpu_tests_pf.log $O/gpu_tests_fl.log
for f in $O/*.json; do echo -n "$f "; python -c "import json,sys; d=json.load(open('$f')); print(d['ms_per_step'], d['phase_ms_per_step']['construct'])"; done
