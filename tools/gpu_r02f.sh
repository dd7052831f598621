# r02f: GPU tests (fused single-block run), A/B of the SM-fill rule, C5 sweep
set -x
O=gpurun_out/r02f; mkdir -p $O
timeout 1500 python -m pytest tests -q -x -m gpu -p no:cacheprovider > $O/gpu_tests.log 2>&1; echo "pytest exit $?" >> $O/gpu_tests.log
B="python bench.py --steps 3 --warmup 3 --parity off --no-cpu-baseline --e2e-steps 1"
for w in c1 c2 c5 c3; do
  ACO_FILL=0 timeout 900 $B --workload $w > $O/${w}_fill0.json 2>$O/${w}_fill0.err
  timeout 900 $B --workload $w > $O/${w}_fill1.json 2>$O/${w}_fill1.err
done
ACO_FUSED_ANTS=0 timeout 600 $B --workload c1 > $O/c1_nofused.json 2>$O/c1_nofused.err
timeout 1500 python tools/c5_sweep.py --steps 3 > $O/c5_sweep.md 2> $O/c5_sweep.err
tail -3 $O/gpu_tests.log
for f in $O/*.json; do echo -n "$f "; python -c "import json,sys; d=json.load(open('$f')); print(d['ms_per_step'], d['phase_ms_per_step']['construct'], d['gpu_launches'])"; done
cat $O/c5_sweep.md
