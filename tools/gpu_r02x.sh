# r02x: fused run with the region state in shared memory (C1) A/B + tests
set -x
O=gpurun_out/r02x; mkdir -p $O
B="python bench.py --steps 5 --warmup 3 --parity off --no-cpu-baseline --e2e-steps 1 --workload c1"
for v in main presrs main presrs; do
  if [ $v = main ]; then unset ACO_LIB_VARIANT; else export ACO_LIB_VARIANT=$v; fi
  timeout 600 $B > $O/c1_$v.json 2>$O/c1.err; mv $O/c1_$v.json $O/c1_${v}_$(date +%s%N).json
done
unset ACO_LIB_VARIANT
timeout 1500 python -m pytest tests -q -x -m gpu -k "fused or fix10a or fig1 or regress or edge" -p no:cacheprovider > $O/gpu_tests.log 2>&1; echo "pytest exit $?" >> $O/gpu_tests.log
tail -2 $O/gpu_tests.log
for f in $O/*.json; do echo -n "$f "; python -c "import json,sys; d=json.load(open('$f')); print(d['ms_per_step'], d['phase_ms_per_step']['construct'])"; done
