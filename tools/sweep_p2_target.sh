#!/bin/bash
# Sweep the pass-2 resident-thread target of the construct launch shapes (C3 batch).
mkdir -p gpurun_out
for t in 384,512 384,640 384,768 384,1024 384,1536 384,768; do
  r=$(ACO_TARGET_THREADS=$t timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['phase_ms_per_step']['construct'])")
  echo "ACO_TARGET_THREADS=$t C3 ms/step construct_ms: $r"
done
