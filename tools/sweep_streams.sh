#!/bin/bash
# Repeat runs of C3 and C5 under ACO_STREAMS 4/5/6/4. The knob is clamped to the 4 internal
# streams (aco_ctx_s::kStreams), so this measures the run-to-run noise floor of the bench.
mkdir -p gpurun_out
for w in c3 c5; do
  for s in 4 5 6 4; do
    r=$(ACO_STREAMS=$s timeout 400 python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'])")
    echo "$w ACO_STREAMS=$s ms/step: $r"
  done
done
