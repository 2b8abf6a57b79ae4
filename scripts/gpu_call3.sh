set -x
make -j8 > /dev/null 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k k_split -s 3 -c 1 -o gpurun_out/prof_k_split_r1b python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full2.log 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_r1.log 2>&1
tail -2 gpurun_out/bench_r1.log
timeout 2400 python scripts/sweep.py --configs C1 C2 C3 C4 --out gpurun_out/sweep_r1.jsonl --table gpurun_out/selector_table_c1c4.json 2>&1 | grep -v Warn | tail -40
timeout 1500 python scripts/sweep.py --configs C5 --classes agg --first-op-only --out gpurun_out/sweep_r1_c5.jsonl 2>&1 | tail -5
