# r02h: C4 global-state lanes / wide per pass; fused run 4-wide (C1)
set -x
O=gpurun_out/r02h; mkdir -p $O
B="python bench.py --steps 3 --warmup 3 --parity off --no-cpu-baseline --e2e-steps 1"
ACO_FUSED_WIDE=0 timeout 600 $B --workload c1 > $O/c1_fw0.json 2>$O/c1_fw0.err
timeout 600 $B --workload c1 > $O/c1_fw1.json 2>$O/c1_fw1.err
for cfg in "16,16 0,0" "16,16 1,0" "16,8 0,0" "16,4 0,0" "16,8 0,1" "16,4 0,1" "8,8 1,0"; do
  set -- $cfg
  ACO_GS_LANES=$1 ACO_GS_WIDE=$2 ACO_GS_WIDE_LANES=16 timeout 900 $B --workload c4 > $O/c4_l${1/,/_}_w${2/,/_}.json 2>$O/c4_l${1/,/_}_w${2/,/_}.err
done
timeout 1200 python -m pytest tests -q -x -m gpu -k "fused or fix10a or global_state or config4" -p no:cacheprovider > $O/gpu_tests.log 2>&1; echo "pytest exit $?" >> $O/gpu_tests.log
tail -3 $O/gpu_tests.log
for f in $O/*.json; do echo -n "$f "; python -c "import json,sys; d=json.load(open('$f')); print(d['ms_per_step'], d['phase_ms_per_step']['construct'])"; done
