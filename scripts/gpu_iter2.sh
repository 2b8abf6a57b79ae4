# usage: bash scripts/gpu_iter2.sh TAG -- full GPU tests, bench, SV sweep on C5 (3 agg classes), ncu
T=${1:-x}
set -x
make -j8 > /dev/null 2>&1
timeout 1500 python -m pytest tests/ -m gpu -x -q 2>&1 | tail -4
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_$T.log 2>&1; tail -c 600 gpurun_out/bench_$T.log
timeout 1200 python scripts/sweep.py --configs C5 --classes agg agg_bin --quick --out gpurun_out/sweep_${T}_c5.jsonl 2>&1 | tail -3
timeout 1200 ncu --set full --clock-control none --import-source on -k k_split -s 3 -c 1 -o gpurun_out/prof_k_split_$T python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-secondary > gpurun_out/ncu_$T.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches_$T.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-secondary > /dev/null 2>&1
