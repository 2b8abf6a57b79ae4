set -x
make -j8 > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_autograd.py -x -q 2>&1 | tail -15
timeout 1500 python scripts/gnn_bench.py --configs C1 C2 C3 --out gpurun_out/gnn_bench_r1.json 2>&1 | tail -20
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/launches_r1j.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-secondary > /dev/null 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k k_split -s 3 -c 1 -o gpurun_out/prof_k_split_r1j python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-secondary > gpurun_out/ncu_r1j.log 2>&1
grep -o '"schedule": "[A-Z0-9_]*"' gpurun_out/ncu_r1j.log | head -1
