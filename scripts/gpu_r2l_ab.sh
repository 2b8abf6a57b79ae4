# round 2 (r2l): 32-bit gather offsets in k_dotsv (UG_DOTSV_O32) and the FMA-folded edge weight
# (UG_MUL_FMA) on the BM 6 / 7 loops
T=${1:-r2l}
C="C4:u_dot_v:128:SV_G64 C3:u_dot_v:128:SV_G64 C4:u_dot_v_sum:128:SV_G64 C4:u_dot_v:256:SV_G128 C5:u_mul_e_sum:602:SV_G2048_F128_P1 C3:u_mul_e_sum:128:SV_G128_F32 C4:u_mul_e_sum:128:SV_G128_F128 C3:copy_u_sum:128:SV_G128_F32"
AB_REPS=30 bash scripts/gpu_ab.sh $T "$C" base "" dotsv64 "-DUG_DOTSV_O32=0" fma "-DUG_MUL_FMA=1"
timeout 900 python -m pytest tests/test_gpu_dotsv.py tests/test_gpu_configs.py -x -q -k "dot" 2>&1 | tail -2
