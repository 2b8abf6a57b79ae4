# usage: bash scripts/gpu_extras.sh TAG -- f4 reordering benchmark + fused GAT probe on the final tree
T=${1:-x}
make -j8 > /dev/null 2>&1
timeout 1200 python scripts/reorder_bench.py > gpurun_out/reorder_$T.log 2>&1; tail -20 gpurun_out/reorder_$T.log
timeout 900 python scripts/gat_probe.py > gpurun_out/gat_$T.log 2>&1; tail -20 gpurun_out/gat_$T.log
