# usage: bash scripts/gpu_sweep.sh TAG -- full schedule sweep (C1-C5) -> sweep jsonl + selector table
T=${1:-r1b}
set -x
make -j8 > /dev/null 2>&1
timeout 3000 python scripts/sweep.py --configs C1 C2 C3 C4 C5 --out gpurun_out/sweep_full_$T.jsonl --table gpurun_out/selector_table_$T.json 2>&1 | grep -v Warn | tail -60
