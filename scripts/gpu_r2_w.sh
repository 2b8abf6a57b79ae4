T=${1:-r2w}
timeout 1500 python scripts/sweep.py --configs C1 C2 --out gpurun_out/sweep_$T.jsonl --table gpurun_out/selector_table_$T.json 2>&1 | grep -v Warn | tail -16
