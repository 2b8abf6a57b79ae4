# round 2 (r2t): k_dotsv register budget of message creation (u_dot_v) with 32-bit offsets: 4 vs 5 CTAs / SM
T=${1:-r2t}
C="C4:u_dot_v:128:SV_G32,SV_G64 C4:u_dot_v:256:SV_G64,SV_G128 C3:u_dot_v:128:SV_G128,SV_G64 C4:u_dot_v_sum:128:SV_G64"
AB_REPS=30 bash scripts/gpu_ab.sh $T "$C" m4 "" m5 "-DUG_DOTSV_MINB_MSG=5"
touch paper_conf_asplos_0001lslwlgslllw23_b200/csrc/k_dotsv.cu; make -j16 EXTRA="-DUG_DOTSV_MINB_MSG=5" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_dotsv.py -x -q 2>&1 | tail -1
touch paper_conf_asplos_0001lslwlgslllw23_b200/csrc/k_dotsv.cu; make -j16 > /dev/null 2>&1
