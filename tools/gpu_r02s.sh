# r02s: A/B the 4-wide / lean size threshold (kWideN 160 vs 128 vs 96)
set -x
O=gpurun_out/r02s; mkdir -p $O
B="python bench.py --steps 3 --warmup 3 --parity off --no-cpu-baseline --e2e-steps 1"
for v in main w128 w96 main; do
  if [ $v = main ]; then unset ACO_LIB_VARIANT; else export ACO_LIB_VARIANT=$v; fi
  timeout 900 $B > $O/c3_$v.json 2>$O/c3_$v.err; mv $O/c3_$v.json $O/c3_${v}_$(date +%s%N).json
done
unset ACO_LIB_VARIANT
for v in w96 w128; do ACO_LIB_VARIANT=$v MB_SIZES=100,130,160 timeout 900 python tools/microbench.py > $O/mb_$v.txt 2>&1; done
MB_SIZES=100,130,160 timeout 900 python tools/microbench.py > $O/mb_main.txt 2>&1
ACO_LIB_VARIANT=w96 timeout 1500 python -m pytest tests -q -x -m gpu -k "every_ant or config2 or lean" -p no:cacheprovider > $O/gpu_tests_w96.log 2>&1; echo "pytest exit $?" >> $O/gpu_tests_w96.log
tail -2 $O/gpu_tests_w96.log
for f in $O/*.json; do echo -n "$f "; python -c "import json,sys; d=json.load(open('$f')); print(d['ms_per_step'], d['phase_ms_per_step']['construct'])"; done
tail -n 3 $O/mb_*.txt
