# timing experiment: how much of u_mul_e_sum's gap to copy_u_sum is the per-edge weight load
T=${1:-r2u}
CASES='C3:u_mul_e_sum:128:SV_G128_F32,SV_G512_F128_P1 C3:copy_u_sum:128:SV_G128_F32 C5:u_mul_e_sum:602:SV_G2048_F128_P1 C5:copy_u_sum:602:SV_G512_F128_P1'
python scripts/ab_sched.py --tag $T-normal --cases $CASES 2>&1
touch paper_conf_asplos_0001lslwlgslllw23_b200/csrc/k_split_mul.cu; make -j16 EXTRA="-DUG_EXPERIMENT_NO_WEIGHT_LOAD" > /dev/null 2>&1
python scripts/ab_sched.py --tag $T-noweightload --cases $CASES 2>&1
touch paper_conf_asplos_0001lslwlgslllw23_b200/csrc/k_split_mul.cu; make -j16 > /dev/null 2>&1
