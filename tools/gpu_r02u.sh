# r02u: huge regions with shared-memory per-ant state (C4) -- A/B + parity
set -x
O=gpurun_out/r02u; mkdir -p $O
timeout 1500 python -m pytest tests -q -x -m gpu -p no:cacheprovider > $O/gpu_tests.log 2>&1; echo "pytest exit $?" >> $O/gpu_tests.log
B="python bench.py --steps 3 --warmup 3 --parity off --no-cpu-baseline --e2e-steps 1"
for r in 1 2; do
  ACO_HUGE_SMEM=0 timeout 900 $B --workload c4 > $O/c4_h0_$r.json 2>$O/c4_h0_$r.err
  timeout 900 $B --workload c4 > $O/c4_h1_$r.json 2>$O/c4_h1_$r.err
done
timeout 900 $B --workload c4 --parity sample > $O/c4_par.json 2>$O/c4_par.err
timeout 900 python bench.py --steps 3 --warmup 3 --workload c4 --e2e-steps 1 > $O/c4_full.json 2>$O/c4_full.err
timeout 900 $B --workload c5 > $O/c5.json 2>$O/c5.err
tail -3 $O/gpu_tests.log
for f in $O/*.json; do echo -n "$f "; python -c "import json,sys; d=json.load(open('$f')); print(d['ms_per_step'], d['phase_ms_per_step']['construct'], d.get('parity') and (d['parity']['bit_exact'], d['parity']['regions']))"; done
