T=${1:-r2s}
timeout 1200 python -m pytest tests/test_gpu_gnn.py tests/test_gpu_dotattn.py tests/test_gpu_autograd.py tests/test_gpu_api.py -x -q 2>&1 | tail -3
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/bench_$T.log 2>&1; tail -c 1500 gpurun_out/bench_$T.log
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:'^k_split$' -s 3 -c 1 -o gpurun_out/prof_k_split_$T python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-secondary > gpurun_out/ncu_$T.log 2>&1; tail -2 gpurun_out/ncu_$T.log
