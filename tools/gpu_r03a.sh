# Session re-entry check of HEAD: GPU tests, smoke, C3 bench.
set -x
O=gpurun_out/r03a; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/gpu.txt
timeout 1500 python -m pytest tests -q -m gpu -x -p no:cacheprovider > $O/gpu_tests.log 2>&1; echo "pytest exit $?" >> $O/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1
timeout 600 python bench.py --steps 5 --warmup 3 > $O/bench_c3.json 2> $O/bench_c3.err
timeout 600 python bench.py --steps 5 --warmup 3 --workload c2 > $O/bench_c2.json 2> $O/bench_c2.err
tail -3 $O/gpu_tests.log; tail -2 $O/smoke.log; cut -c1-300 $O/bench_c3.json $O/bench_c2.json
