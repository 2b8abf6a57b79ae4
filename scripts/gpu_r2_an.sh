# round 2: column-index prefetch (the next group's col_idx loads overlap this group's row
# gathers: one dependent L2 round trip per group instead of two) in the SV fast loop
# (UG_PF_BM2 / UG_PF_BM0) and the dot-attention traversals (UG_DA_PF)
T=${1:-r2an}
CS=paper_conf_asplos_0001lslwlgslllw23_b200/csrc
CASES='C4:u_dot_v:128:SV_G64 C3:u_dot_v:128:SV_G64 C4:u_dot_v_sum:128:SV_G64 C3:u_mul_e_sum:128:SV_G128_F32,SV_G128_F64 C3:u_mul_e_sum:32:SV_G128_F32 C2:u_mul_e_sum:64:SV_G16_F64 C5:u_mul_e_sum:602:SV_G2048_F128_P1 C3:copy_u_sum:128:SV_G128_F32 C5:copy_u_sum:602:SV_G512_F128_P1'
variant() {
  touch $CS/k_split*.cu $CS/k_dotattn.cu $CS/k_dotsv.cu; make -j16 EXTRA="$2" > /dev/null 2>&1 || { echo "build $1 failed"; return; }
  echo "== $1 ($2)"
  timeout 900 python scripts/ab_sched.py --tag $T-$1 --cases $CASES 2>&1 | grep '^{'
  timeout 600 python scripts/dotattn_probe.py --tag $T-$1 2>&1 | grep '^{'
}
variant pf0 "-DUG_PF_BM2=0 -DUG_DA_PF=0 -DUG_DOTSV_PF=0"
variant pf1 "-DUG_PF_BM2=1 -DUG_DA_PF=1"
variant pf1uf8 "-DUG_PF_BM2=1 -DUG_BM2_UF=8 -DUG_BM2_SUM_MINB=5"
variant pf1m5 "-DUG_PF_BM2=1 -DUG_BM2_SUM_MINB=5"
variant bm0pf6 "-DUG_PF_BM0=1 -DUG_BM0_MINB=6"
variant bm0pf7 "-DUG_PF_BM0=1 -DUG_BM0_MINB=7"
touch $CS/k_split*.cu $CS/k_dotattn.cu $CS/k_dotsv.cu; make -j16 > /dev/null 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_dotattn.py -x -q 2>&1 | tail -2
