set -x
O=gpurun_out/r03o; mkdir -p $O
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
ACO_SYNC_DEBUG=1 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_coverage.py tests/test_gpu_lpi.py -x -q -p no:cacheprovider > $O/tests.log 2>&1; echo "pytest exit $?" >> $O/tests.log
tail -3 $O/tests.log
for i in 1 2; do MATRIX="c1" BM_OUT=$O bash tools/bench_matrix.sh >> $O/matrix.log 2>&1; done
cut -c1-250 $O/matrix.log
