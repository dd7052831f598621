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
if [ -n "$PROF_TOP" ]; then
  export PROF_ITERS=1
  timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"${TOP_RE:-k_construct<.int.2, .int.1, .bool.1, .bool.0}" -c 1 -o gpurun_out/prof_top python tools/prof_run.py > gpurun_out/prof_top.log 2>&1
fi
