set -x
make -j8 > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "SV or strided or padding" 2>&1 | tail -2
for S in SV_G128_F64_P1 SV_G512_F64_P1 SV_G128_F128_P1 SV_G512_F128_P1; do python scripts/prof_op.py --config C5 --op copy_u_sum --F 602 --schedule $S --reps 5; done
UG_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --steps 3 --warmup 3 > gpurun_out/dry2.log 2>&1; echo "rc=$?"; tail -c 1500 gpurun_out/dry2.log
UG_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29512 bench.py --gpus 2 --steps 3 --warmup 3 --op u_mul_e_sum > gpurun_out/dry2b.log 2>&1; echo "rc=$?"; tail -c 800 gpurun_out/dry2b.log
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29513 bench.py --impl reference --gpus 2 --steps 3 --warmup 3 > gpurun_out/dry2c.log 2>&1; echo "rc=$?"; tail -c 400 gpurun_out/dry2c.log
