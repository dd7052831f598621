set -x
O=gpurun_out/r03i; mkdir -p $O
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
ACO_SYNC_DEBUG=1 ACO_GRAPH=0 timeout 120 python tools/repro_lpi.py > $O/sync.log 2>&1; grep -a "aco sync\|ok\|Error" $O/sync.log | head
ACO_SYNC_DEBUG=1 ACO_GRAPH=0 ACO_LPI=0 timeout 120 python tools/repro_lpi.py > $O/sync0.log 2>&1; grep -a "aco sync\|ok\|Error" $O/sync0.log | head
ACO_SYNC_DEBUG=1 ACO_GRAPH=0 SIZES=3,5 timeout 120 python tools/repro_lpi.py > $O/sync35.log 2>&1; grep -a "aco sync\|ok\|Error" $O/sync35.log | head
ACO_SYNC_DEBUG=1 ACO_GRAPH=0 SIZES=11,13 timeout 120 python tools/repro_lpi.py > $O/sync1113.log 2>&1; grep -a "aco sync\|ok\|Error" $O/sync1113.log | head
