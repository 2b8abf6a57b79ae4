# usage: bash scripts/gpu_iter.sh TAG  -- parity subset, bench, C5 SV sweep, ncu of k_split
T=${1:-x}
set -x
make -j8 > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -3
timeout 900 python -m pytest tests/test_gpu_configs.py -x -q -k "C5_headline or C5_padded or sharded or C3_schedule" 2>&1 | tail -3
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_$T.log 2>&1; tail -c 3000 gpurun_out/bench_$T.log
timeout 1200 python scripts/sweep.py --configs C5 --classes agg --first-op-only --quick --out gpurun_out/sweep_${T}_c5.jsonl 2>&1 | tail -2
timeout 1200 ncu --set full --clock-control none --import-source on -k k_split -s 3 -c 1 -o gpurun_out/prof_k_split_$T python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-secondary > gpurun_out/ncu_$T.log 2>&1
