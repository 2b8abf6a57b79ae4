set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -5
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "not all_ops_all_schedules" 2>&1 | tail -30
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "all_ops_all_schedules" 2>&1 | tail -30
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline 2>&1 | tail -5
