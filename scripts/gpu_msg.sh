# usage: bash scripts/gpu_msg.sh -- SV message-creation fast path: parity + timings vs the TE/WE schedules
make -j8 > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -k "message_creation_sv or all_ops_all_schedules and add" -x -q 2>&1 | tail -3
for a in "C3 u_add_v 32" "C4 u_add_v 128" "C2 u_add_v 64"; do
  set -- $a
  for S in TE_G8_T4 WE_G16_T1 TE_G4_T8 SV_G16_F32 SV_G64_F32 SV_G128_F32 SV_G32_F64 SV_G64_F128 SV_G512_F128; do
    timeout 300 python scripts/prof_op.py --config $1 --op $2 --F $3 --schedule $S --reps 20
  done
done
