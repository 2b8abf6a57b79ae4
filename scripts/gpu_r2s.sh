# round 2 (r2s): k_dott register budget after the full-tile / 32-bit-offset loop: 6 vs 8 CTAs / SM
T=${1:-r2s}
CS=paper_conf_asplos_0001lslwlgslllw23_b200/csrc
C="C5:u_dot_v:602:SV_G256_F128,SV_G512_F128 C5:u_dot_v_sum:602:SV_G256_F128 C3:u_dot_v:128:SV_G256_F128 C4:u_dot_v:256:SV_G128_F128 C5:copy_u_sum:602:SV_G512_F128_P1"
for m in 6 8 7; do
  touch $CS/k_dott.cu; make -j16 EXTRA="-DUG_DOTT_MINB=$m" > gpurun_out/build_$T-$m.log 2>&1 || { echo "build $m failed"; continue; }
  echo "== minb$m"
  timeout 900 python -m pytest tests/test_gpu_dott.py -x -q 2>&1 | tail -1
  timeout 900 python scripts/ab_sched.py --tag $T-minb$m --reps 20 --cases $C 2>&1 | grep '^{'
done
touch $CS/k_dott.cu; make -j16 > /dev/null 2>&1
