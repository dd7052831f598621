# New defaults (huge shared-state path, bulk staging, one-launch finalize): GPU tests + bench lines.
set -x
O=gpurun_out/r03k; mkdir -p $O
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
timeout 1500 python -m pytest tests -q -m gpu -p no:cacheprovider > $O/gpu_tests.log 2>&1; echo "pytest exit $?" >> $O/gpu_tests.log
tail -5 $O/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; tail -2 $O/smoke.log
MATRIX="c4 c5 c2 c1 c3" BM_OUT=$O bash tools/bench_matrix.sh > $O/matrix.log 2>&1
cut -c1-250 $O/matrix.log
