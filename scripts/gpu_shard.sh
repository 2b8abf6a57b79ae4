# round 2: the N > 1 path on one GPU -- world-2 gloo parity vs the oracle, then a torchrun dry run
T=${1:-r2a}
nproc; lscpu | grep 'Model name'
timeout 1800 python -m pytest tests/test_gpu_sharded.py -x -q 2>&1 | tail -15
UG_DIST_BACKEND=gloo timeout 1200 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
  --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 5 --warmup 3 \
  > gpurun_out/bench_dry2_$T.log 2>&1; tail -c 2500 gpurun_out/bench_dry2_$T.log
