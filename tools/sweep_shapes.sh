# Launch-shape knob sweep on the C3 bench (run under gpurun): ms per step and phases.
# SWEEP="thr1,thr2:lanes1,lanes2 ..." (targets of resident threads per SM, max lanes per ant, pass 1,2)
for cfg in ${SWEEP:-512,256:8,1 512,512:8,1 1024,512:8,1 512,768:8,1 1024,1024:8,1 512,512:4,1 512,512:8,4}; do
  t=${cfg%%:*}; l=${cfg##*:}
  echo "== threads $t lanes $l"
  ACO_TARGET_THREADS=$t ACO_MAX_LANES=$l timeout 300 python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['phase_ms_per_step'], d['gpu_launches'])"
done
