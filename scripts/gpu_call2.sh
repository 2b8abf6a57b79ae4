set -x
make -j8 > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "not all_ops_all_schedules" 2>&1 | tail -15
timeout 2000 python -m pytest tests/test_gpu_configs.py -x -q --durations=15 2>&1 | tail -40
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/launches_r1.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_launch_bench.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_split -s 3 -c 1 -o gpurun_out/prof_k_split_r1 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full.log 2>&1
tail -3 gpurun_out/ncu_full.log
