timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
BENCH_DIST_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 20 --warmup 3 --no-cpu-baseline 2>&1 | grep -E "^\{|Error|error" | cut -c1-400
