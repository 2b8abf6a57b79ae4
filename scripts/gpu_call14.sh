set -x
make -j8 > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_api.py tests/test_gpu_parity.py -x -q 2>&1 | tail -3
for S in SV_G128_F64_P1 SV_G128_F32; do python scripts/prof_op.py --config C5 --op u_mul_e_sum --F 602 --schedule $S --reps 3; done
timeout 3000 python scripts/sweep.py --configs C1 C2 C3 C4 C5 --out gpurun_out/sweep_full_r1b.jsonl --table gpurun_out/selector_table_r1b.json 2>&1 | grep -v Warn | grep -E "^C|wrote"
