# round 2: register-budget A/B of k_dotsv (UG_DOTSV_MINB) and k_dotattn_heads (UG_DAH_MINB);
# ncu r2ac showed 64 / 70 registers and 45 % / 34 % warps active.
T=${1:-r2ad}
CS=paper_conf_asplos_0001lslwlgslllw23_b200/csrc
CASES='C4:u_dot_v:128:SV_G256_F128,WE_G4_T1 C3:u_dot_v:128:SV_G256_F128 C2:u_dot_v:64:SV_G256_F128 C4:u_dot_v_sum:128:SV_G256_F128'
variant() {
  touch $CS/k_dotsv.cu $CS/k_dotattn.cu; make -j16 EXTRA="$2" > /dev/null 2>&1 || { echo "build $1 failed"; return; }
  echo "== $1 ($2)"
  timeout 600 python scripts/ab_sched.py --tag $T-$1 --cases $CASES 2>&1 | tail -8
  timeout 600 python scripts/gat_probe.py 2>&1 | grep dot_attention
}
variant base ""
variant dotsv5 "-DUG_DOTSV_MINB=5"
variant dah3 "-DUG_DAH_MINB=3"
variant dah4 "-DUG_DAH_MINB=4"
touch $CS/k_dotsv.cu $CS/k_dotattn.cu; make -j16 > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_dotattn.py tests/test_gpu_dott.py -x -q 2>&1 | tail -2
