set -x
O=gpurun_out/r03n; mkdir -p $O
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
timeout 900 python -m pytest tests/test_gpu_lpi.py tests/test_gpu_parity.py -x -q -p no:cacheprovider > $O/tests.log 2>&1; echo "pytest exit $?" >> $O/tests.log
tail -3 $O/tests.log
MATRIX="c2" BM_OUT=$O bash tools/bench_matrix.sh > $O/matrix.log 2>&1
cut -c1-250 $O/matrix.log
