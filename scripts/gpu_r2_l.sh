T=${1:-r2l}
timeout 900 python -m pytest tests/test_gpu_dott.py -x -q 2>&1 | tail -2
CASES='C5:u_dot_v:602:SV_G512_F64,SV_G512_F128,SV_G2048_F128 C4:u_dot_v:256:SV_G64,SV_G256_F128 C4:u_dot_v:128:SV_G64,SV_G256_F128 C5:u_dot_v_sum:602:SV_G512_F128'
timeout 900 python scripts/ab_sched.py --tag $T-default --cases $CASES 2>&1
touch paper_conf_asplos_0001lslwlgslllw23_b200/csrc/k_dott.cu
make -j16 EXTRA="-DUG_DOTT_PIPE4=1 -DUG_DOTT_MINB=3" > /dev/null 2>&1
timeout 900 python scripts/ab_sched.py --tag $T-pipe4-minb3 --cases $CASES 2>&1
touch paper_conf_asplos_0001lslwlgslllw23_b200/csrc/k_dott.cu
make -j16 EXTRA="-DUG_DOTT_MINB=5" > /dev/null 2>&1
timeout 900 python scripts/ab_sched.py --tag $T-minb5 --cases $CASES 2>&1
