#!/bin/bash
# C1 (64 ants, one 10-instruction region) under the spread launch shapes.
mkdir -p gpurun_out
for e in ACO_X=0 ACO_SPREAD=1 "ACO_SPREAD=1 ACO_SPREAD_CAP=8" "ACO_SPREAD=1 ACO_SPREAD_CAP=1" ACO_X=0; do
  r=$(env $e timeout 300 python bench.py --workload c1 --steps 5 --warmup 3 --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['phase_ms_per_step'])")
  echo "c1 $e: $r"
done
