set -x
make -j8 > /dev/null 2>&1
timeout 3000 python scripts/sweep.py --configs C1 C2 C3 C4 C5 --out gpurun_out/sweep_full_r1.jsonl --table gpurun_out/selector_table_r1.json 2>&1 | grep -v Warn | tail -60
