# usage: bash scripts/gpu_ab.sh TAG -- SV chunk order A/B (UG_SV_ORDER=row vs longest-first) + parity subset
T=${1:-x}
make -j8 > /dev/null 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_configs.py tests/test_gpu_gat.py tests/test_gpu_arg.py -x -q 2>&1 | tail -3
for ORD in row len; do
  echo "== order $ORD"
  export UG_SV_ORDER=$ORD
  for a in "C3 copy_u_sum 32 SV_G32_F32" "C3 copy_u_sum 32 SV_G16_F32" "C3 copy_u_sum 64 SV_G32_F64" "C3 copy_u_sum 128 SV_G32_F128" \
           "C3 u_mul_e_sum 32 SV_G32_F32" "C3 u_mul_e_sum 128 SV_G32_F128_P1" "C3 copy_u_max 128 SV_G32_F128" \
           "C4 copy_u_sum 128 SV_G32_F128" "C2 u_mul_e_sum 64 SV_G16_F64" "C3 copy_u_sum 128 SV_G32_F32" "C3 copy_u_sum 128 SV_G64_F32"; do
    set -- $a
    timeout 300 python scripts/prof_op.py --config $1 --op $2 --F $3 --schedule $4 --reps 20
  done
  timeout 600 python scripts/probe_c5.py --reps 6 2>&1 | tail -5
done
