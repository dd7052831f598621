# r02 profile: GPU tests, C3 launch list, ncu --set full of the first iteration's
# launches, source capture of the top pass-2 class, the C4 global-state kernels.
set -x
O=gpurun_out/r02c; mkdir -p $O
timeout 1200 python -m pytest tests -q -m gpu -p no:cacheprovider > $O/gpu_tests.log 2>&1; echo "pytest exit $?" >> $O/gpu_tests.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --parity off --e2e-steps 1 > $O/launches_bench.log 2>&1
export PROF_ITERS=1
timeout 1200 ncu --set full --clock-control none -k regex:'k_construct|k_select|k_update' -c 60 -o /tmp/prof_all python tools/prof_run.py > $O/prof_all.log 2>&1
ncu -i /tmp/prof_all.ncu-rep --page raw --csv > $O/prof_raw.csv 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"k_construct<.int.2, .int.1, .bool.1, .bool.0, .bool.0, .bool.0, .int.2, .bool.1, .bool.1>" -c 1 -o $O/prof_top python tools/prof_run.py > $O/prof_top.log 2>&1
ncu -i $O/prof_top.ncu-rep --page source --csv --print-source cuda,sass > $O/prof_top_source.csv 2>/dev/null
ncu -i $O/prof_top.ncu-rep --page raw --csv > $O/prof_top_raw.csv 2>/dev/null
PROBE_N=2000 PROBE_ITERS=1 timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:k_construct -c 2 -o $O/prof_gs python tools/size_probe.py > $O/prof_gs.log 2>&1
ncu -i $O/prof_gs.ncu-rep --page raw --csv > $O/prof_gs_raw.csv 2>/dev/null
ncu -i $O/prof_gs.ncu-rep --page source --csv --print-source cuda,sass > $O/prof_gs_source.csv 2>/dev/null
rm -f $O/*.ncu-rep
ls -la $O; du -sh $O
tail -3 $O/gpu_tests.log
