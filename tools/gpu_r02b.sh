# A/B: global-state per-ant layout (ant-major vs [word][ant]) + lane-parallel init
set -x
mkdir -p gpurun_out/r02b
ACO_LIB_VARIANT=gsam timeout 1200 python -m pytest tests -q -x -m gpu -p no:cacheprovider > gpurun_out/r02b/gpu_tests_gsam.log 2>&1
tail -3 gpurun_out/r02b/gpu_tests_gsam.log
for w in c4 c5; do
  timeout 600 python bench.py --workload $w --steps 3 --warmup 3 --parity off --no-cpu-baseline > gpurun_out/r02b/${w}_base.json 2>gpurun_out/r02b/${w}_base.err
  ACO_LIB_VARIANT=gsam ACO_GS_LAYOUT=0 timeout 600 python bench.py --workload $w --steps 3 --warmup 3 --parity off --no-cpu-baseline > gpurun_out/r02b/${w}_gsam0.json 2>>gpurun_out/r02b/${w}_gsam.err
  ACO_LIB_VARIANT=gsam ACO_GS_LAYOUT=1 timeout 600 python bench.py --workload $w --steps 3 --warmup 3 --parity off --no-cpu-baseline > gpurun_out/r02b/${w}_gsam1.json 2>>gpurun_out/r02b/${w}_gsam.err
done
for w in c1 c2; do
  timeout 600 python bench.py --workload $w --steps 5 --warmup 3 > gpurun_out/r02b/${w}_base.json 2>gpurun_out/r02b/${w}_base.err
done
for f in gpurun_out/r02b/*.json; do echo $f; python -c "import json,sys; d=json.load(open('$f')); print(d['ms_per_step'], d['phase_ms_per_step'], d.get('parity') and d['parity']['bit_exact'])"; done
