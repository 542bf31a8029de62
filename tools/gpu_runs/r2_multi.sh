# the N > 1 bench path on the one-GPU box: 2 ranks share GPU 0 over gloo (IRR_BENCH_DIST_BACKEND=gloo),
# strong scaling (the config's batch LPT-split over the ranks), status words all-gathered
export IRR_BENCH_DIST_BACKEND=gloo
for c in C3 C5; do
  timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29517 \
     bench.py --gpus 2 --config $c --steps 3 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/bench_multi2_$c.json 2> gpurun_out/bench_multi2_$c.err
  echo "$c rc=$?"; tail -c 600 gpurun_out/bench_multi2_$c.json
done
