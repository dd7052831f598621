for cfg in "512,256 8,1" "768,256 8,1" "512,192 4,1" "512,128 2,1" "384,256 4,1" "512,256 8,2" "1024,256 8,1"; do
  set -- $cfg
  echo "== threads $1 lanes $2"
  ACO_TARGET_THREADS=$1 ACO_MAX_LANES=$2 timeout 300 python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['phase_ms_per_step'])"
done
