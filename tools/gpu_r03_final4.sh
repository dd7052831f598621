# r03 final verification of the last build: GPU tests, smoke, bench matrix
# (every line parity-checked), C3 parity over every region, ncu evidence with
# the build fingerprint (-> profiles/r03_traffic.json), C2 lane-per-instruction
# and C4 huge-region captures, C5 per-n sweep, Table-6 analogue.
# (compute-sanitizer is closed on this pool since r03: not run.)
set -x
O=gpurun_out/r03final4; mkdir -p $O
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,driver_version --format=csv > $O/gpu.txt
lscpu | grep -i "model name\|^CPU(s)" > $O/host.txt
timeout 1500 python -m pytest tests -q -m gpu --durations=15 -p no:cacheprovider > $O/gpu_tests.log 2>&1; echo "pytest exit $?" >> $O/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1
BM_OUT=$O/matrix bash tools/bench_matrix.sh > $O/matrix.log 2>&1
timeout 1500 python bench.py --steps 3 --warmup 3 --parity all --parity-log $O/parity_all_c3.log > $O/bench_c3_parity_all.json 2> $O/bench_c3_parity_all.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --parity off --e2e-steps 1 > $O/launches_bench.log 2>&1
export PROF_ITERS=1
timeout 1200 ncu --set full --clock-control none -k regex:'k_construct|k_select|k_update' -c 60 -o /tmp/prof_all python tools/prof_run.py > $O/prof_all.log 2>&1
ncu -i /tmp/prof_all.ncu-rep --page raw --csv > $O/prof_raw.csv 2>&1
FP=$(python -c "from paper_conf_cgo_shobakimhlmkrg24_b200 import build as B; print(B.source_fingerprint())")
python tools/ncu_table.py $O/prof_raw.csv $O/r03_traffic.json "profiles/r03_final4/prof_raw.csv: ncu --set full, first iteration of both passes of the C3 batch, dram__bytes_read.sum + dram__bytes_write.sum averaged over the construct launches" $FP > $O/ncu_table.md
timeout 600 ncu --set full --clock-control none -k regex:'k_construct|k_finalize1' -c 6 -o /tmp/prof_c2 python tools/prof_c2.py > $O/prof_c2.log 2>&1
ncu -i /tmp/prof_c2.ncu-rep --page raw --csv > $O/prof_c2_raw.csv 2>/dev/null
PROBE_N=2000 PROBE_ITERS=1 timeout 900 ncu --set full --clock-control none -k regex:k_construct -c 2 -o /tmp/prof_gs python tools/size_probe.py > $O/prof_c4.log 2>&1
ncu -i /tmp/prof_gs.ncu-rep --page raw --csv > $O/prof_c4_raw.csv 2>/dev/null
timeout 1200 python tools/c5_sweep.py > $O/c5_sweep.md 2> $O/c5_sweep.err
rm -f /tmp/*.ncu-rep
tail -3 $O/gpu_tests.log; tail -2 $O/smoke.log; cut -c1-200 $O/matrix.log; head -c 300 $O/bench_c3_parity_all.json
