# usage: bash scripts/gpu_bench.sh TAG -- default bench line + GNN end-to-end benchmark
T=${1:-x}
make -j8 > /dev/null 2>&1
timeout 900 python bench.py > gpurun_out/bench_$T.log 2>&1; tail -c 300 gpurun_out/bench_$T.log
timeout 900 python scripts/gnn_bench.py --configs C1 C2 C3 --out gpurun_out/gnn_bench_$T.json 2>&1 | tail -25
