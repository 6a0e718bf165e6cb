# Functional check of bench.py's N = 2 flow (torchrun, max-over-ranks timing, rank-0 JSON)
# on a one-GPU box: both ranks share cuda:0 and talk over gloo.  Not a performance number.
for mode in sharded peer replicas; do
  STG_BENCH_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
    --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 2 --warmup 3 --config C4 --mode $mode \
    --no-cpu-baseline > gpurun_out/bench_n2_$mode.log 2>&1
  echo "$mode rc=$?"; tail -1 gpurun_out/bench_n2_$mode.log | cut -c1-400
done
