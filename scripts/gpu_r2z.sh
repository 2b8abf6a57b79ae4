# round 2 (r2z): SV tail -- one predicated full-size group for a remainder > UF / 2 (UG_SV_TAIL_FULL)
T=${1:-r2z}
CS=paper_conf_asplos_0001lslwlgslllw23_b200/csrc
C="C3:copy_u_sum:128:SV_G128_F32 C3:u_mul_e_sum:128:SV_G128_F64 C3:copy_u_sum:32:SV_G128_F32 C3:copy_u_max:128:SV_G128_F32 C4:copy_u_sum:128:SV_G128_F128_P1 C4:u_mul_e_sum:128:SV_G128_F128 C2:u_mul_e_sum:64:SV_G16_F64 C2:copy_u_sum:64:SV_G16_F64 C5:copy_u_sum:602:SV_G512_F128_P1 C5:u_mul_e_sum:602:SV_G512_F128_P1"
for m in 0 1; do
  touch $CS/k_split*.cu; make -j16 EXTRA="-DUG_SV_TAIL_FULL=$m" > gpurun_out/build_$T-$m.log 2>&1 || { echo "build $m failed"; continue; }
  echo "== tail$m"
  if [ $m = 1 ]; then timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bm67.py tests/test_gpu_configs.py -x -q -k "sv or non_power or contiguous or C3 or C4 or C2 or C1 or C5_headline" 2>&1 | tail -1; fi
  timeout 900 python scripts/ab_sched.py --tag $T-tail$m --reps 30 --cases $C 2>&1 | grep '^{'
done
touch $CS/k_split*.cu; make -j16 > /dev/null 2>&1
