# Line-level evidence for C2 (one warp per SM, latency-bound) and the top C3 classes.
set -x
O=gpurun_out/r03b; mkdir -p $O
for ps in 1 3; do PROF_TIME=1 PROF_ITERS=100 PROF_PASSES=$ps timeout 300 python tools/prof_c2.py >> $O/c2_time.log 2>&1; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_construct -c 4 -o $O/c2 python tools/prof_c2.py > $O/c2_prof.log 2>&1
ncu -i $O/c2.ncu-rep --page source --csv --print-source cuda,sass > $O/c2_source.csv 2>/dev/null
ncu -i $O/c2.ncu-rep --page raw --csv > $O/c2_raw.csv 2>/dev/null
export PROF_ITERS=1
for re in "k_construct<.int.2, .int.1, .bool.1, .bool.0, .bool.0, .bool.0, .int.0, .bool.1, .bool.1>" "k_construct<.int.1, .int.1, .bool.1, .bool.0, .bool.0, .bool.0, .int.0, .bool.1, .bool.0>"; do
  tag=$(echo "$re" | tr -dc '0-9' | cut -c1-12)
  timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"$re" -c 1 -o $O/c3_$tag python tools/prof_run.py > $O/c3_$tag.log 2>&1
  ncu -i $O/c3_$tag.ncu-rep --page source --csv --print-source cuda,sass > $O/c3_${tag}_source.csv 2>/dev/null
done
rm -f $O/*.ncu-rep
ls -la $O; cat $O/c2_time.log
