# round 2: register budgets of k_dotattn (wide, UG_DAW_MINB), k_dotattn_heads (UG_DAH_MINB) and
# k_dotsv (UG_DOTSV_MINB, schedules SV_Gg without a column tile)
T=${1:-r2ae}
CS=paper_conf_asplos_0001lslwlgslllw23_b200/csrc
CASES='C4:u_dot_v:128:SV_G64,SV_G128 C4:u_dot_v:256:SV_G128 C3:u_dot_v:128:SV_G64 C2:u_dot_v:64:SV_G64 C4:u_dot_v_sum:128:SV_G64'
variant() {
  touch $CS/k_dotsv.cu $CS/k_dotattn.cu; make -j16 EXTRA="$2" > /dev/null 2>&1 || { echo "build $1 failed"; return; }
  echo "== $1 ($2)"
  timeout 600 python scripts/ab_sched.py --tag $T-$1 --cases $CASES 2>&1 | tail -6
  timeout 600 python scripts/dotattn_probe.py --tag $T-$1 2>&1
}
variant base ""
variant v5 "-DUG_DOTSV_MINB=5 '-DUG_DAH_MINB=(VEC==4?4:5)' '-DUG_DAW_MINB=(VEC==4?3:4)'"
variant v6 "-DUG_DOTSV_MINB=6 '-DUG_DAH_MINB=(VEC==4?5:6)' -DUG_DAW_MINB=4"
touch $CS/k_dotsv.cu $CS/k_dotattn.cu; make -j16 > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_dotattn.py -x -q 2>&1 | tail -2
