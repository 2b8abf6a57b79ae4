# usage: bash scripts/gpu_libab.sh LIB... -- time the same ops against alternative builds (UG_LIBRARY)
for L in "$@"; do
  echo "== lib $L"
  export UG_LIBRARY=$PWD/$L
  for a in "C3 copy_u_sum 32 SV_G128_F32" "C3 copy_u_sum 32 SV_G32_F32" "C3 copy_u_sum 128 SV_G128_F32" "C3 u_mul_e_sum 32 SV_G128_F32" \
           "C3 u_mul_e_sum 128 SV_G512_F128_P1" "C4 copy_u_sum 128 SV_G128_F128_P1" "C2 u_mul_e_sum 64 SV_G16_F64" "C3 copy_u_max 128 SV_G128_F64_P1"; do
    set -- $a
    timeout 300 python scripts/prof_op.py --config $1 --op $2 --F $3 --schedule $4 --reps 20
  done
  timeout 600 python scripts/probe_c5.py --reps 6 2>&1 | grep -E "^(b2b|gap) " | head -2
done
