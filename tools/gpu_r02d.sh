# A/B round: packed kill tests (mk) for the lean layout, GS 4-wide scan, CUDA graph replay
set -x
O=gpurun_out/r02d; mkdir -p $O
timeout 1200 python -m pytest tests -q -x -m gpu -p no:cacheprovider > $O/gpu_tests.log 2>&1; echo "pytest exit $?" >> $O/gpu_tests.log
B="python bench.py --steps 3 --warmup 3 --parity off --no-cpu-baseline --e2e-steps 1"
ACO_LIB_VARIANT=gsam timeout 600 $B > $O/c3_old.json 2>$O/c3_old.err
ACO_GRAPH=0 timeout 600 $B > $O/c3_nograph.json 2>$O/c3_nograph.err
timeout 600 $B > $O/c3_new.json 2>$O/c3_new.err
for w in c1 c2; do
  ACO_GRAPH=0 timeout 600 $B --workload $w > $O/${w}_nograph.json 2>$O/${w}_nograph.err
  timeout 600 $B --workload $w > $O/${w}_graph.json 2>$O/${w}_graph.err
done
for w in c4 c5; do
  ACO_GS_WIDE=0 timeout 600 $B --workload $w > $O/${w}_gs1.json 2>$O/${w}_gs1.err
  timeout 600 $B --workload $w > $O/${w}_gs4.json 2>$O/${w}_gs4.err
done
tail -3 $O/gpu_tests.log
for f in $O/*.json; do echo $f; python -c "import json,sys; d=json.load(open('$f')); print(d['ms_per_step'], d['phase_ms_per_step']['construct'], d['gpu_launches'])"; done
