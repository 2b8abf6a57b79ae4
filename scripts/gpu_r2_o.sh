T=${1:-r2o}
timeout 900 python -m pytest tests/test_gpu_dotattn.py tests/test_gpu_concurrency.py -x -q 2>&1 | tail -2
python scripts/gat_probe.py 2>&1 | tail -1 > gpurun_out/gat_probe_$T.json; cat gpurun_out/gat_probe_$T.json
timeout 4800 python scripts/sweep.py --configs C1 C2 C3 C4 C5 --out gpurun_out/sweep_$T.jsonl --table gpurun_out/selector_table_$T.json 2>&1 | grep -v Warn | tail -40
