# r02z: R24 prune with the critical-path bound (ACO_PRUNE_CP) A/B + parity with it on
set -x
O=gpurun_out/r02z; mkdir -p $O
ACO_PRUNE_CP=1 timeout 1500 python -m pytest tests -q -x -m gpu -p no:cacheprovider > $O/gpu_tests_pcp.log 2>&1; echo "pytest exit $?" >> $O/gpu_tests_pcp.log
B="python bench.py --steps 3 --warmup 3 --parity off --no-cpu-baseline --e2e-steps 1"
for v in 0 1 0 1; do ACO_PRUNE_CP=$v timeout 900 $B > $O/c3_$v.json 2>$O/c3.err; mv $O/c3_$v.json $O/c3_${v}_$(date +%s%N).json; done
for w in c2 c5 c4; do for v in 0 1; do ACO_PRUNE_CP=$v timeout 900 $B --workload $w > $O/${w}_$v.json 2>$O/$w.err; done; done
ACO_PRUNE_CP=1 timeout 900 python bench.py --steps 3 --warmup 3 --e2e-steps 1 > $O/c3_pcp_parity.json 2>$O/c3p.err
tail -2 $O/gpu_tests_pcp.log
for f in $O/*.json; do echo -n "$f "; python -c "import json,sys; d=json.load(open('$f')); print(d['ms_per_step'], d['phase_ms_per_step']['construct'], d['pruned_pass2_ant_frac'], d.get('parity') and d['parity']['bit_exact'])"; done
