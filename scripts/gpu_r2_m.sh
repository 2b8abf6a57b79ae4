T=${1:-r2m}
timeout 900 python -m pytest tests/test_gpu_dott.py -x -q 2>&1 | tail -2
CASES='C5:u_dot_v:602:SV_G512_F128,SV_G2048_F128,SV_G256_F128 C4:u_dot_v:256:SV_G256_F128 C4:u_dot_v:128:SV_G256_F128 C5:u_dot_v_sum:602:SV_G2048_F128 C5:copy_u_sum:602:SV_G512_F128_P1'
timeout 900 python scripts/ab_sched.py --tag $T-minb5 --cases $CASES 2>&1
touch paper_conf_asplos_0001lslwlgslllw23_b200/csrc/k_dott.cu
make -j16 EXTRA="-DUG_DOTT_MINB=6" > /dev/null 2>&1
timeout 900 python scripts/ab_sched.py --tag $T-minb6 --cases $CASES 2>&1
touch paper_conf_asplos_0001lslwlgslllw23_b200/csrc/k_dott.cu; make -j16 > /dev/null 2>&1
# C1 latency: device duration of each kernel (ncu) vs the CUDA-event latency
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:'^k_' --csv --log-file gpurun_out/ncu_c1_$T.csv \
  python scripts/ab_sched.py --reps 3 --cases "C1:u_mul_e_sum:16:TE_G1_T16,SV_G16_F16,SV_G8_F16,BV_G1_B256" "C2:copy_u_max:8:SV_G16_F16,WE_G4_T1" > /dev/null 2>&1
python scripts/ab_sched.py --reps 20 --cases "C1:u_mul_e_sum:16:TE_G1_T16,SV_G16_F16,SV_G8_F16,BV_G1_B256" "C2:copy_u_max:8:SV_G16_F16,WE_G4_T1" 2>&1
