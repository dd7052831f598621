# r02n: general machine model (R42) in the compact layout (was u32 cycles only)
set -x
O=gpurun_out/r02n; mkdir -p $O
timeout 1500 python -m pytest tests -q -x -m gpu -p no:cacheprovider > $O/gpu_tests.log 2>&1; echo "pytest exit $?" >> $O/gpu_tests.log
B="python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1"
timeout 900 $B --machine dual > $O/c3_dual.json 2>$O/c3_dual.err
timeout 900 $B --machine dual --parity sample --cpu-sample 48 > $O/c3_dual_par.json 2>$O/c3_dual_par.err
timeout 900 $B > $O/c3.json 2>$O/c3.err
tail -3 $O/gpu_tests.log
for f in $O/*.json; do echo -n "$f "; python -c "import json,sys; d=json.load(open('$f')); print(d['ms_per_step'], d['phase_ms_per_step']['construct'], d.get('parity'))"; done
