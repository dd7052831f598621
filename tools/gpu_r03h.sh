set -x
O=gpurun_out/r03h; mkdir -p $O
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
for i in 0 1 2 3 4 5 6 7 8 9 10 11 12 13; do echo "size idx $i: $(SIZES=$i timeout 60 python tools/repro_lpi.py 2>&1 | tail -1)" >> $O/bisect.log; done
echo "lpi0: $(ACO_LPI=0 timeout 60 python tools/repro_lpi.py 2>&1 | tail -1)" >> $O/bisect.log
echo "all again: $(timeout 60 python tools/repro_lpi.py 2>&1 | tail -1)" >> $O/bisect.log
echo "mode1: $(MODE=1 timeout 60 python tools/repro_lpi.py 2>&1 | tail -1)" >> $O/bisect.log
echo "nodump: $(DUMP=0 timeout 60 python tools/repro_lpi.py 2>&1 | tail -1)" >> $O/bisect.log
cat $O/bisect.log
