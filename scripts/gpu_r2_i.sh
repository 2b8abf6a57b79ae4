# round 2: parity suite after the SV merge / dott changes, then per-op A/B of the touched paths
T=${1:-r2i}
timeout 2400 python -m pytest tests/ -m gpu -x -q 2>&1 | tail -4
timeout 900 python scripts/ab_sched.py --tag $T --cases \
  "C3:copy_u_sum:128:SV_G128_F32,SV_G512_F128_P1" "C3:u_mul_e_sum:128:SV_G512_F128_P1" "C3:copy_u_sum:32:SV_G128_F32" \
  "C2:copy_u_max:8:SV_G16_F16,SV_G32_F16,WE_G4_T1" "C2:u_mul_e_sum:64:SV_G16_F64,SV_G32_F64" \
  "C1:u_mul_e_sum:16:TE_G1_T16,SV_G16_F16,SV_G32_F16,SV_G8_F16,SV_G64_F16,BV_G1_B256" \
  "C1:copy_u_sum:16:BV_G1_B256,SV_G16_F16,SV_G32_F16" \
  "C5:copy_u_sum:602:SV_G512_F128_P1" "C5:u_dot_v:602:SV_G512_F128,SV_G2048_F128" 2>&1 | tee gpurun_out/ab_$T.jsonl
