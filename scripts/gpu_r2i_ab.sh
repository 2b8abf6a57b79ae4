# round 2 (r2i): SV fast loop with a contiguous per-edge scalar weight (BM 6: pointer + immediate
# addressing, no per-edge offset registers) vs the generic edge-scalar mode (BM 2), at its register
# budgets / gathers in flight; then the C1 / C2 sweep with the edge-lanes TV schedules
T=${1:-r2i}
M="C3:u_mul_e_sum:128:SV_G128_F32,SV_G128_F64,SV_G128_F128 C3:u_mul_e_sum:32:SV_G128_F32 C4:u_mul_e_sum:128:SV_G128_F128,SV_G128_F32 C2:u_mul_e_sum:64:SV_G16_F64 C5:u_mul_e_sum:602:SV_G2048_F128_P1,SV_G512_F128_P1 C3:copy_u_sum:128:SV_G128_F32 C5:copy_u_sum:602:SV_G512_F128_P1"
AB_REPS=30 bash scripts/gpu_ab.sh $T "$M" bm2 "-DUG_SV_BM6=0" bm6 "" bm6uf8 "-DUG_BM6_UF=8" bm6uf8m8 "-DUG_BM6_UF=8 -DUG_BM6_SUM_MINB=8" bm6m8 "-DUG_BM6_SUM_MINB=8"
timeout 1500 python -m pytest tests/test_gpu_configs.py tests/test_gpu_views_r2.py tests/test_gpu_edgelanes.py -x -q -k "mul or edgelanes or view or sv" 2>&1 | tail -2
timeout 900 python scripts/sweep.py --configs C1 C2 --reps 40 --out gpurun_out/sweep_${T}_C1C2.jsonl --table gpurun_out/selector_table_${T}_C1C2.json 2>&1 | grep -v Warn | tail -14
