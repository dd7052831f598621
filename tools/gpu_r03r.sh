# Source-level ncu capture of the final build's lane-per-instruction ants (C2) and the top C3 classes.
set -x
O=gpurun_out/r03r; mkdir -p $O
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_construct -c 2 -o $O/c2 python tools/prof_c2.py > $O/c2_prof.log 2>&1
ncu -i $O/c2.ncu-rep --page source --csv --print-source cuda,sass > $O/c2_source.csv 2>/dev/null
export PROF_ITERS=1
for re in "k_construct<.int.2, .int.1, .bool.1, .bool.0, .bool.0, .bool.0, .int.2, .bool.1, .bool.1>" "k_construct<.int.1, .int.1, .bool.1, .bool.0, .bool.0, .bool.0, .int.0, .bool.1, .bool.0>"; do
  tag=$(echo "$re" | tr -dc '0-9' | cut -c1-12)
  timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"$re" -c 1 -o $O/c3_$tag python tools/prof_run.py > $O/c3_$tag.log 2>&1
  ncu -i $O/c3_$tag.ncu-rep --page source --csv --print-source cuda,sass > $O/c3_${tag}_source.csv 2>/dev/null
done
rm -f $O/*.ncu-rep
for f in $O/*_source.csv; do echo "== $f"; python tools/src_lines.py $f 30 > ${f%.csv}_lines.txt; head -5 ${f%.csv}_lines.txt; done
rm -f $O/*_source.csv
