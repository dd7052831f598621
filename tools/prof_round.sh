# ncu evidence for one round (run under gpurun; writes gpurun_out/):
#  launches.csv  : launch list of the bench command (gpu__time_duration per launch)
#  prof_raw.csv  : every metric of --set full for every construct/select/update
#                  launch of the first iteration of both passes (report not kept: size)
#  prof_top.ncu-rep : full capture with source of the top pass-1 and pass-2 classes
set -x
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py
if [ -z "$SKIP_LAUNCHES" ]; then
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/launches_bench.log 2>&1
fi
export PROF_ITERS=1
timeout 900 ncu --set full --clock-control none -k regex:'k_construct|k_select|k_update' -c ${PROF_COUNT:-40} -o /tmp/prof_all python tools/prof_run.py > gpurun_out/prof_all.log 2>&1
ncu -i /tmp/prof_all.ncu-rep --page raw --csv > gpurun_out/prof_raw.csv 2>&1
ncu -i /tmp/prof_all.ncu-rep --page details --csv > gpurun_out/prof_details.csv 2>&1
timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"${TOP_RE:-k_construct<.int.2, .int.1, .bool.1, .bool.0}" -c 1 -o gpurun_out/prof_top python tools/prof_run.py > gpurun_out/prof_top.log 2>&1
ls -la gpurun_out
du -sh gpurun_out
