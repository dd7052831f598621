set -x
O=gpurun_out/r03j; mkdir -p $O
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py nobulk ACO_BULK_STAGE=0 > /dev/null
echo "default: $(ACO_SYNC_DEBUG=1 timeout 120 python tools/repro_lpi.py 2>&1 | grep -a 'aco sync\|^ok' | head -3)" >> $O/r.log
echo "nofin1: $(ACO_FIN1=0 ACO_SYNC_DEBUG=1 timeout 120 python tools/repro_lpi.py 2>&1 | grep -a 'aco sync\|^ok' | head -3)" >> $O/r.log
echo "nobulk: $(ACO_LIB_VARIANT=nobulk ACO_SYNC_DEBUG=1 timeout 120 python tools/repro_lpi.py 2>&1 | grep -a 'aco sync\|^ok' | head -3)" >> $O/r.log
cat $O/r.log
timeout 1500 python -m pytest tests -q -m gpu -p no:cacheprovider > $O/gpu_tests.log 2>&1; echo "pytest exit $?" >> $O/gpu_tests.log
tail -5 $O/gpu_tests.log
