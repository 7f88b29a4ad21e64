# Functional check of the N > 1 bench path on a 1-GPU box (ranks share the GPU, gloo all-reduce):
# the driver's scaling run uses the same code with NCCL on one GPU per rank.
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29531 \
  bench.py --gpus 2 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_n2.json 2> gpurun_out/bench_n2.err
echo "rc=$?"; tail -c 400 gpurun_out/bench_n2.json; tail -5 gpurun_out/bench_n2.err
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29532 \
  bench.py --impl reference --gpus 2 --steps 1 --warmup 3 > gpurun_out/bench_ref_n2.json 2> gpurun_out/bench_ref_n2.err
echo "rc=$?"; head -c 300 gpurun_out/bench_ref_n2.json
for c in c2 c3; do timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_$c.json 2>/dev/null; head -c 260 gpurun_out/bench_$c.json; echo; done
