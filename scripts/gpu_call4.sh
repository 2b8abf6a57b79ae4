set -x
make -j8 > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -5
timeout 900 python -m pytest tests/test_gpu_configs.py -x -q -k "C5_headline or C5_padded or sharded or C3_schedule" 2>&1 | tail -5
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_r1d.log 2>&1; tail -1 gpurun_out/bench_r1c.log
timeout 1200 python scripts/sweep.py --configs C5 --classes agg --first-op-only --quick --out gpurun_out/sweep_r1d_c5.jsonl 2>&1 | tail -3
timeout 1200 python scripts/sweep.py --configs C3 --classes agg --out gpurun_out/sweep_r1d_c3.jsonl 2>&1 | tail -12
timeout 1200 ncu --set full --clock-control none --import-source on -k k_split -s 3 -c 1 -o gpurun_out/prof_k_split_r1d python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full4.log 2>&1
