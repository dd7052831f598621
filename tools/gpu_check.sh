# One GPU verification round (run under gpurun): build, GPU tests, bench,
# optional launch-shape A/B on the per-size microbenchmark.
set -x
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py
timeout 1200 python -m pytest tests -x -q -m gpu 2>&1 | tail -15 | tee gpurun_out/gpu_tests.log
timeout 600 python bench.py --steps 3 --warmup 3 2>&1 | tail -1 | tee gpurun_out/bench.log
for lanes in ${AB_LANES:-}; do
  echo "== ACO_MAX_LANES_WIDE=$lanes" | tee -a gpurun_out/ab.log
  ACO_MAX_LANES_WIDE=$lanes MB_SIZES=${MB_SIZES:-250,450} timeout 400 python tools/microbench.py 2>&1 | tee -a gpurun_out/ab.log
done
