# multi-rank code paths on ONE GPU (gloo; not a performance number): LD (triangle plan with the
# chunked overlapped broadcast) and FastID (db shards, query broadcast, packed-key best merge)
for w in ld2k fastid1m; do
  BENCH_DIST_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
    --master-addr 127.0.0.1 --master-port 29533 bench.py --workload $w --gpus 2 --steps 5 --warmup 3 \
    --no-cpu-baseline 2>&1 | grep -E "^\{|Error|error" | cut -c1-600
done
