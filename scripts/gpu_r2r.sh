# round 2 (r2r): column-index staging in the SV fast loop (UG_SV_IDX_STAGE: 1 = cp.async,
# 2 = 1-D bulk TMA + mbarrier) against the register-index loop (0), on the L = 32 schedules
T=${1:-r2r}
CS=paper_conf_asplos_0001lslwlgslllw23_b200/csrc
C="C5:copy_u_sum:602:SV_G512_F128_P1 C5:u_mul_e_sum:602:SV_G512_F128_P1 C4:copy_u_sum:128:SV_G128_F128 C4:u_mul_e_sum:128:SV_G128_F128 C3:copy_u_sum:128:SV_G128_F128 C3:u_mul_e_sum:128:SV_G128_F128"
for m in 0 1 2; do
  touch $CS/k_split*.cu; make -j16 EXTRA="-DUG_SV_IDX_STAGE=$m" > gpurun_out/build_$T-$m.log 2>&1 || { echo "build $m failed"; continue; }
  echo "== stage$m"
  timeout 1200 python -m pytest tests/test_gpu_configs.py -x -q -k "C5_headline or C5_padded or C4 or C3" 2>&1 | tail -1
  timeout 900 python scripts/ab_sched.py --tag $T-stage$m --reps 20 --cases $C 2>&1 | grep '^{'
done
touch $CS/k_split*.cu; make -j16 > /dev/null 2>&1
