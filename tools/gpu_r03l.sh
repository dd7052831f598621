set -x
O=gpurun_out/r03l; mkdir -p $O
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
ACO_SYNC_DEBUG=1 timeout 600 python -m pytest tests/test_gpu_lpi.py -x -q -p no:cacheprovider > $O/lpi_tests.log 2>&1; echo "pytest exit $?" >> $O/lpi_tests.log
tail -20 $O/lpi_tests.log
timeout 1500 python -m pytest tests -q -m gpu -p no:cacheprovider > $O/gpu_tests.log 2>&1; echo "pytest exit $?" >> $O/gpu_tests.log
tail -5 $O/gpu_tests.log
MATRIX="c1 c2" BM_OUT=$O bash tools/bench_matrix.sh > $O/matrix.log 2>&1
cut -c1-250 $O/matrix.log
