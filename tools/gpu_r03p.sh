# r03p: dry run of bench.py's N > 1 paths on one GPU (two ranks on cuda:0, gloo)
set -x
O=gpurun_out/r03p; mkdir -p $O
export ACO_BENCH_ONE_GPU=1 ACO_BENCH_BACKEND=gloo
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --steps 2 --warmup 3 --regions 600 > $O/c3_n2.json 2> $O/c3_n2.err
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29512 bench.py --gpus 2 --steps 2 --warmup 3 --regions 600 --scaling weak > $O/c3_n2_weak.json 2> $O/c3_n2_weak.err
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29513 bench.py --gpus 2 --steps 2 --warmup 3 --workload c4 --ants 2048 --iterations 2 > $O/c4_n2.json 2> $O/c4_n2.err
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29514 bench.py --gpus 2 --steps 2 --warmup 3 --workload c5 --iterations 2 > $O/c5_n2.json 2> $O/c5_n2.err
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29515 bench.py --gpus 2 --steps 2 --warmup 3 --impl reference --cpu-sample 32 > $O/ref_n2.json 2> $O/ref_n2.err
for f in $O/*.json; do echo "== $f"; head -c 1200 $f; echo; tail -3 ${f%.json}.err; done
export ACO_BENCH_ONE_GPU=1 ACO_BENCH_BACKEND=gloo
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29516 bench.py --gpus 2 --steps 2 --warmup 3 --workload c2 --iterations 10 > gpurun_out/r03p/c2_n2.json 2> gpurun_out/r03p/c2_n2.err
head -c 600 gpurun_out/r03p/c2_n2.json
