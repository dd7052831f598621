# r02w: re-tune pass-1 shape knobs on the final kernels (max lanes of wide classes, thread targets)
set -x
O=gpurun_out/r02w; mkdir -p $O
B="python bench.py --steps 3 --warmup 3 --parity off --no-cpu-baseline --e2e-steps 1"
run() { tag=$1; shift; env "$@" timeout 900 $B > $O/c3_$tag.json 2>$O/c3_$tag.err; }
run base
run mlw1 ACO_MAX_LANES_WIDE=1,1
run mlw2 ACO_MAX_LANES_WIDE=2,1
run t320 ACO_TARGET_THREADS=320,768
run t448 ACO_TARGET_THREADS=448,768
run t512 ACO_TARGET_THREADS=512,768
run p2_512 ACO_TARGET_THREADS=384,512
run p2_1024 ACO_TARGET_THREADS=384,1024
run base2
for f in $O/*.json; do echo -n "$f "; python -c "import json,sys; d=json.load(open('$f')); print(d['ms_per_step'], d['phase_ms_per_step']['construct'])"; done
