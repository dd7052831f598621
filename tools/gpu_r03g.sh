set -x
O=gpurun_out/r03g; mkdir -p $O
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py nobulk ACO_BULK_STAGE=0 > /dev/null
timeout 120 python tools/repro_lpi.py > $O/default.log 2>&1; tail -2 $O/default.log
ACO_FIN1=0 timeout 120 python tools/repro_lpi.py > $O/nofin1.log 2>&1; tail -2 $O/nofin1.log
ACO_LIB_VARIANT=nobulk timeout 120 python tools/repro_lpi.py > $O/nobulk.log 2>&1; tail -2 $O/nobulk.log
DUMP=0 timeout 120 python tools/repro_lpi.py > $O/nodump.log 2>&1; tail -2 $O/nodump.log
timeout 600 compute-sanitizer --tool memcheck --print-limit 20 python tools/repro_lpi.py > $O/memcheck.log 2>&1; head -60 $O/memcheck.log
