# Source-level ncu captures of the construct kernels on equal-size batches.
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py
export PROF_ITERS=1
for cfg in ${PROF_CFGS:-400:300:1 400:300:2 60:2000:2}; do
  n=${cfg%%:*}; rest=${cfg#*:}; r=${rest%%:*}; p=${rest##*:}
  PROF_N=$n PROF_REGIONS=$r timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
    -k regex:"k_construct<.int.$p" -c 1 -o gpurun_out/prof_n${n}_p$p python tools/prof_run.py > gpurun_out/prof_n${n}_p$p.log 2>&1
done
ls -la gpurun_out; du -sh gpurun_out
