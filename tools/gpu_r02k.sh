# r02k: final verification of a build: GPU tests, smoke, the bench matrix,
# ncu evidence (launch list, --set full of the first iteration, top-class source)
# with the build fingerprint -> profiles/r02_traffic.json
set -x
O=gpurun_out/r02k; mkdir -p $O
timeout 1500 python -m pytest tests -q -m gpu -p no:cacheprovider > $O/gpu_tests.log 2>&1; echo "pytest exit $?" >> $O/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1
BM_OUT=$O/matrix bash tools/bench_matrix.sh > $O/matrix.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --parity off --e2e-steps 1 > $O/launches_bench.log 2>&1
export PROF_ITERS=1
timeout 1200 ncu --set full --clock-control none -k regex:'k_construct|k_select|k_update' -c 60 -o /tmp/prof_all python tools/prof_run.py > $O/prof_all.log 2>&1
ncu -i /tmp/prof_all.ncu-rep --page raw --csv > $O/prof_raw.csv 2>&1
FP=$(python -c "from paper_conf_cgo_shobakimhlmkrg24_b200 import build as B; print(B.source_fingerprint())")
python tools/ncu_table.py $O/prof_raw.csv $O/r02_traffic.json "profiles/r02_final/prof_raw.csv: ncu --set full, first iteration of both passes of the C3 batch, dram__bytes_read.sum + dram__bytes_write.sum averaged over the construct launches" $FP > $O/ncu_table.md
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"k_construct<.int.2, .int.1, .bool.1, .bool.0, .bool.0, .bool.0, .int.2, .bool.1, .bool.1>" -c 1 -o $O/prof_top python tools/prof_run.py > $O/prof_top.log 2>&1
ncu -i $O/prof_top.ncu-rep --page source --csv --print-source cuda,sass > $O/prof_top_source.csv 2>/dev/null
ncu -i $O/prof_top.ncu-rep --page raw --csv > $O/prof_top_raw.csv 2>/dev/null
rm -f $O/*.ncu-rep
tail -3 $O/gpu_tests.log; cat $O/smoke.log | tail -2; cat $O/matrix.log
