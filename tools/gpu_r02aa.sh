# r02aa: few large regions -- global-state kernels instead of under-filled shared-memory blocks?
set -x
O=gpurun_out/r02aa; mkdir -p $O
timeout 900 python tools/c5_sweep.py --steps 3 --sizes 500,1000 > $O/sweep_base.md 2>$O/e1
ACO_GS_MIN_THREADS=4096,4096 timeout 900 python tools/c5_sweep.py --steps 3 --sizes 500,1000 > $O/sweep_gs.md 2>$O/e2
B="python bench.py --steps 3 --warmup 3 --parity off --no-cpu-baseline --e2e-steps 1 --workload c5"
timeout 900 $B > $O/c5_base.json 2>$O/e3
ACO_GS_MIN_THREADS=4096,4096 timeout 900 $B > $O/c5_gs.json 2>$O/e4
cat $O/sweep_base.md $O/sweep_gs.md
for f in $O/*.json; do echo -n "$f "; python -c "import json,sys; d=json.load(open('$f')); print(d['ms_per_step'], d['phase_ms_per_step']['construct'])"; done
