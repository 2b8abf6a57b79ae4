set -x
make -j8 > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_gnn.py -x -q 2>&1 | tail -15
timeout 1200 python scripts/gnn_bench.py --configs C1 C2 C3 --out gpurun_out/gnn_bench_r1.json 2>&1 | tail -20
timeout 900 python bench.py > gpurun_out/bench_r1i.log 2>&1; tail -c 300 gpurun_out/bench_r1i.log
