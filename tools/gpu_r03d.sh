# Source-level profile of the lane-per-instruction ants (C2) and the fused C1 run.
set -x
O=gpurun_out/r03d; mkdir -p $O
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_construct -c 4 -o $O/c2 python tools/prof_c2.py > $O/c2_prof.log 2>&1
ncu -i $O/c2.ncu-rep --page source --csv --print-source cuda,sass > $O/c2_source.csv 2>/dev/null
ncu -i $O/c2.ncu-rep --page raw --csv > $O/c2_raw.csv 2>/dev/null
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_fused -c 1 -o $O/c1 python bench.py --workload c1 --steps 1 --warmup 0 --no-cpu-baseline --parity off --e2e-steps 1 > $O/c1_prof.log 2>&1
ncu -i $O/c1.ncu-rep --page source --csv --print-source cuda,sass > $O/c1_source.csv 2>/dev/null
ncu -i $O/c1.ncu-rep --page raw --csv > $O/c1_raw.csv 2>/dev/null
rm -f $O/*.ncu-rep
ls -la $O
