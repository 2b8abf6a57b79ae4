# usage: bash scripts/gpu_libab3.sh LIB... -- SV message creation (u_add_v) against alternative builds
for L in "$@"; do
  echo "== lib $L"
  export UG_LIBRARY=$PWD/$L
  for a in "C3 u_add_v 32 SV_G16_F32" "C3 u_add_v 32 SV_G64_F32" "C4 u_add_v 128 SV_G32_F64" "C4 u_add_v 128 SV_G16_F32" "C2 u_add_v 64 SV_G16_F32"; do
    set -- $a
    timeout 300 python scripts/prof_op.py --config $1 --op $2 --F $3 --schedule $4 --reps 20
  done
done
