# Round-2 GPU verification: GPU tests (with durations), smoke, C3 bench line.
set -x
mkdir -p gpurun_out/r02a
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r02a/gpu.txt
timeout 1500 python -m pytest tests -q -m gpu --durations=25 -p no:cacheprovider > gpurun_out/r02a/gpu_tests.log 2>&1
echo "pytest exit $?" >> gpurun_out/r02a/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02a/smoke.log 2>&1
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/r02a/bench_c3.json 2> gpurun_out/r02a/bench_c3.err
tail -3 gpurun_out/r02a/gpu_tests.log
cat gpurun_out/r02a/bench_c3.json | head -c 3000
