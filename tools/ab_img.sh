# A/B: block image staged in shared memory vs read through L1 (ACO_IMG_L1 per pass)
python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
for v in 0,0 1,1; do
  echo "== ACO_IMG_L1=$v"
  ACO_IMG_L1=$v MB_SIZES=${MB_SIZES:-120,200,300,450} timeout 400 python tools/microbench.py
done
timeout 900 python -m pytest tests -x -q -m gpu 2>&1 | tail -3
for v in 0,0 1,1; do
  echo "== bench ACO_IMG_L1=$v"
  ACO_IMG_L1=$v timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | cut -c1-400
done
