# r02v: C2 (one region, latency-bound): 4-wide thresholds
set -x
O=gpurun_out/r02v; mkdir -p $O
B="python bench.py --steps 3 --warmup 3 --parity off --no-cpu-baseline --e2e-steps 1 --workload c2"
for t in 160,120 160,96 160,64 96,96 64,64 160,120; do ACO_WIDE_N=$t timeout 900 $B > $O/c2_$t.json 2>$O/c2.err; mv $O/c2_$t.json $O/c2_${t/,/_}_$(date +%s%N).json; done
for f in $O/*.json; do echo -n "$f "; python -c "import json,sys; d=json.load(open('$f')); print(d['ms_per_step'], d['phase_ms_per_step']['construct'])"; done
