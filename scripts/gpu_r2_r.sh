# round 2: width-1 weight vector rule + FMA / register-budget A/B for u_mul_e_sum
T=${1:-r2r}
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_configs.py -x -q -k "mul or strided or C5" 2>&1 | tail -2
CASES='C5:u_mul_e_sum:602:SV_G512_F64_P1,SV_G512_F128_P1,SV_G128_F128_P1,SV_G2048_F128_P1,SV_G512_F64_P1_V2 C3:u_mul_e_sum:128:SV_G128_F32,SV_G128_F64_V2,SV_G128_F32_V2,SV_G512_F128_P1 C5:copy_u_sum:602:SV_G512_F128_P1'
python scripts/ab_sched.py --tag $T-default --cases $CASES 2>&1
touch paper_conf_asplos_0001lslwlgslllw23_b200/csrc/k_split_mul.cu; make -j16 EXTRA="-DUG_MUL_FMA=1" > /dev/null 2>&1
python scripts/ab_sched.py --tag $T-fma --cases $CASES 2>&1
touch paper_conf_asplos_0001lslwlgslllw23_b200/csrc/k_split_mul.cu; make -j16 EXTRA="-DUG_MUL_FMA=1 -DUG_BM2_SUM_MINB=8" > /dev/null 2>&1
python scripts/ab_sched.py --tag $T-fma-minb8 --cases $CASES 2>&1
touch paper_conf_asplos_0001lslwlgslllw23_b200/csrc/k_split_mul.cu; make -j16 > /dev/null 2>&1
