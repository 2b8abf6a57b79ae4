# usage: bash scripts/gpu_power.sh -- C5 copy_u_sum schedules under sustained back-to-back load (power cap)
make -j8 > /dev/null 2>&1
for S in SV_G512_F128_P1 SV_G128_F64_P1 SV_G512_F64_P1 SV_G2048_F128_P1 SV_G512_F32_P1; do
  timeout 300 python scripts/probe_c5.py --schedule $S --reps 30 --modes b2b 2>&1 | tail -2
done
