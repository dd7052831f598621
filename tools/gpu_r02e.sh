# r02e: sanitizers, Table-6 analogue, C5 per-n sweep, C3 parity over every region
set -x
O=gpurun_out/r02e; mkdir -p $O
bash tools/gpu_sanitize.sh > $O/sanitize_summary.txt 2>&1
timeout 900 python tools/table6.py > $O/table6.md 2> $O/table6.err
timeout 1500 python tools/c5_sweep.py --steps 3 > $O/c5_sweep.md 2> $O/c5_sweep.err
timeout 1500 python bench.py --steps 3 --warmup 3 --parity all --parity-log $O/parity_all_c3.log > $O/bench_c3_parity_all.json 2> $O/bench_c3_parity_all.err
cat $O/table6.md; cat $O/c5_sweep.md; head -c 600 $O/bench_c3_parity_all.json; grep -c ok $O/parity_all_c3.log
