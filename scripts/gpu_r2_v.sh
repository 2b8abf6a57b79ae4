T=${1:-r2v}
timeout 900 python -m pytest tests/test_gpu_edgelanes.py tests/test_gpu_dotattn.py -x -q 2>&1 | tail -2
python scripts/ab_sched.py --reps 20 --tag $T --cases "C1:u_mul_e_sum:16:TE_G1_T4,WV_G1_T1_E1,WV_G4_T1_E1,WV_G2_T1_E1" "C1:copy_u_sum:16:TE_G1_T4,WV_G1_T1_E1,WV_G4_T1_E1" "C1:copy_u_max:16:BV_G1_B256,WV_G1_T1_E1,WV_G4_T1_E1" "C2:copy_u_max:8:SV_G16_F16,WV_G1_T1_E1,WV_G4_T1_E1" "C2:copy_u_sum:8:WE_G4_T1,WV_G1_T1_E1,WV_G4_T1_E1" "C2:u_mul_e_sum:64:SV_G16_F64" "C2:copy_u_sum:64:SV_G16_F64" "C3:copy_u_sum:32:SV_G128_F32,WV_G1_T1_E1" 2>&1
