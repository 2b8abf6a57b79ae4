# usage: bash scripts/gpu_libab2.sh LIB... -- u_mul_e_sum (B = scalar edge weight) against alternative builds
for L in "$@"; do
  echo "== lib $L"
  export UG_LIBRARY=$PWD/$L
  for a in "C3 u_mul_e_sum 128 SV_G512_F64_P1" "C3 u_mul_e_sum 128 SV_G128_F32" "C3 u_mul_e_sum 32 SV_G128_F32" \
           "C4 u_mul_e_sum 128 SV_G512_F128_P1" "C4 u_mul_e_sum 128 SV_G128_F32" "C2 u_mul_e_sum 64 SV_G16_F64"; do
    set -- $a
    timeout 300 python scripts/prof_op.py --config $1 --op $2 --F $3 --schedule $4 --reps 20
  done
done
