# Lane-per-instruction ants: parity tests first, then the whole GPU suite, C2 bench.
set -x
O=gpurun_out/r03c; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_lpi.py -x -q -p no:cacheprovider > $O/lpi_tests.log 2>&1; echo "pytest exit $?" >> $O/lpi_tests.log
tail -30 $O/lpi_tests.log
timeout 1500 python -m pytest tests -q -m gpu -p no:cacheprovider > $O/gpu_tests.log 2>&1; echo "pytest exit $?" >> $O/gpu_tests.log
tail -15 $O/gpu_tests.log
timeout 600 python bench.py --steps 5 --warmup 3 --workload c2 > $O/bench_c2.json 2> $O/bench_c2.err
cut -c1-400 $O/bench_c2.json; tail -3 $O/bench_c2.err
for ps in 1 3; do PROF_TIME=1 PROF_ITERS=100 PROF_PASSES=$ps timeout 300 python tools/prof_c2.py >> $O/c2_time.log 2>&1; done
cat $O/c2_time.log
