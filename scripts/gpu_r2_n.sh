T=${1:-r2n}
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_gat.py tests/test_gpu_arg.py tests/test_gpu_concurrency.py tests/test_gpu_nan.py -x -q 2>&1 | tail -2
python scripts/ab_sched.py --reps 20 --tag $T --cases "C1:u_mul_e_sum:16:TE_G1_T16,SV_G16_F16,SV_G8_F16,SV_G4_F16" "C1:copy_u_sum:16:BV_G1_B256,SV_G16_F16,SV_G8_F16" "C2:copy_u_max:8:SV_G16_F16,SV_G8_F16,WE_G4_T1" "C2:u_mul_e_sum:64:SV_G16_F64,SV_G8_F64" 2>&1
python scripts/gat_probe.py 2>&1 | tail -3
