# r02p: source-level ncu captures of the top pass-1 class and the staged lean pass-2 class
set -x
O=gpurun_out/r02p; mkdir -p $O
export PROF_ITERS=1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"k_construct<.int.1, .int.1, .bool.1, .bool.0, .bool.0, .bool.0, .int.0, .bool.1, .bool.0>" -c 1 -o $O/p1 python tools/prof_run.py > $O/p1.log 2>&1
ncu -i $O/p1.ncu-rep --page source --csv --print-source cuda,sass > $O/p1_source.csv 2>/dev/null
ncu -i $O/p1.ncu-rep --page raw --csv > $O/p1_raw.csv 2>/dev/null
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"k_construct<.int.2, .int.1, .bool.1, .bool.0, .bool.0, .bool.0, .int.0, .bool.1, .bool.1>" -c 1 -o $O/p2s python tools/prof_run.py > $O/p2s.log 2>&1
ncu -i $O/p2s.ncu-rep --page source --csv --print-source cuda,sass > $O/p2s_source.csv 2>/dev/null
ncu -i $O/p2s.ncu-rep --page raw --csv > $O/p2s_raw.csv 2>/dev/null
rm -f $O/*.ncu-rep; ls -la $O
