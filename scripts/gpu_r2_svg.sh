# round 2: staged SV (k_svg: "_M1" TMA gather4, "_A1" cp.async) -- parity, then A/B against the
# register SV kernel (k_split)
T=${1:-r2c}
timeout 1200 python -m pytest tests/test_gpu_svg.py tests/test_gpu_concurrency.py tests/test_gpu_reorder.py -x -q 2>&1 | tail -5
timeout 900 python scripts/ab_sched.py --tag $T --cases \
  "C3:u_mul_e_sum:128:SV_G512_F128_P1,SV_G512_F128_A1,SV_G128_F128_A1,SV_G128_F64_A1,SV_G512_F128_M1,SV_G128_F128_M1" \
  "C3:copy_u_sum:128:SV_G128_F32,SV_G512_F128_A1,SV_G128_F128_A1,SV_G128_F64_A1,SV_G128_F32_A1,SV_G128_F128_M1" \
  "C3:u_mul_e_sum:32:SV_G128_F32,SV_G128_F32_A1,SV_G128_F32_M1" \
  "C3:copy_u_sum:32:SV_G128_F32,SV_G128_F32_A1,SV_G128_F32_M1" \
  "C4:u_mul_e_sum:128:SV_G128_F128,SV_G128_F128_A1,SV_G128_F128_M1" \
  "C4:copy_u_sum:128:SV_G128_F128,SV_G128_F128_A1,SV_G128_F128_M1" \
  "C5:copy_u_sum:602:SV_G512_F128_P1,SV_G512_F128_P1_A1,SV_G512_F128_P1_M1" \
  "C5:u_mul_e_sum:602:SV_G512_F64_P1,SV_G512_F128_P1_A1,SV_G512_F128_P1_M1" \
  2>&1 | tee gpurun_out/ab_$T.jsonl
