set -x
make -j8 > /dev/null 2>&1
timeout 2400 python scripts/sweep.py --configs C5 C3 --classes agg agg_bin agg_ext --out gpurun_out/sweep_c5c3_r1c.jsonl --table gpurun_out/selector_table_c5c3_r1c.json 2>&1 | grep -E "^C|wrote"
