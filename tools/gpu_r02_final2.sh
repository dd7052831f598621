# r02 final verification of the last build: GPU tests, smoke, bench matrix,
# C3 parity over every region, ncu evidence with the build fingerprint,
# sanitizers on every case.
set -x
O=gpurun_out/final2; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,driver_version --format=csv > $O/gpu.txt
timeout 1500 python -m pytest tests -q -m gpu --durations=15 -p no:cacheprovider > $O/gpu_tests.log 2>&1; echo "pytest exit $?" >> $O/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1
BM_OUT=$O/matrix bash tools/bench_matrix.sh > $O/matrix.log 2>&1
timeout 1500 python bench.py --steps 3 --warmup 3 --parity all --parity-log $O/parity_all_c3.log > $O/bench_c3_parity_all.json 2> $O/bench_c3_parity_all.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --parity off --e2e-steps 1 > $O/launches_bench.log 2>&1
export PROF_ITERS=1
timeout 1200 ncu --set full --clock-control none -k regex:'k_construct|k_select|k_update' -c 60 -o /tmp/prof_all python tools/prof_run.py > $O/prof_all.log 2>&1
ncu -i /tmp/prof_all.ncu-rep --page raw --csv > $O/prof_raw.csv 2>&1
FP=$(python -c "from paper_conf_cgo_shobakimhlmkrg24_b200 import build as B; print(B.source_fingerprint())")
python tools/ncu_table.py $O/prof_raw.csv $O/r02_traffic.json "profiles/r02_final/prof_raw.csv: ncu --set full, first iteration of both passes of the C3 batch, dram__bytes_read.sum + dram__bytes_write.sum averaged over the construct launches" $FP > $O/ncu_table.md
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"k_construct<.int.2, .int.1, .bool.1, .bool.0, .bool.0, .bool.0, .int.2, .bool.1, .bool.1>" -c 1 -o $O/prof_top python tools/prof_run.py > $O/prof_top.log 2>&1
ncu -i $O/prof_top.ncu-rep --page source --csv --print-source cuda,sass > $O/prof_top_source.csv 2>/dev/null
ncu -i $O/prof_top.ncu-rep --page raw --csv > $O/prof_top_raw.csv 2>/dev/null
PROBE_N=2000 PROBE_ITERS=1 timeout 900 ncu --set full --clock-control none -k regex:k_construct -c 2 -o $O/prof_gs python tools/size_probe.py > $O/prof_gs.log 2>&1
ncu -i $O/prof_gs.ncu-rep --page raw --csv > $O/prof_gs_raw.csv 2>/dev/null
rm -f $O/*.ncu-rep
rm -rf gpurun_out/sanitize; bash tools/gpu_sanitize.sh > $O/sanitize_summary.txt 2>&1
cp -r gpurun_out/sanitize $O/sanitize
tail -3 $O/gpu_tests.log; tail -2 $O/smoke.log; cat $O/matrix.log | cut -c1-200; head -c 300 $O/bench_c3_parity_all.json
