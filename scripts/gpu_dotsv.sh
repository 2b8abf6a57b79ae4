# usage: bash scripts/gpu_dotsv.sh -- k_dotsv parity + timings vs the edge-unit dot kernel
make -j8 > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_dotsv.py -x -q 2>&1 | tail -3
for a in "C4 u_dot_v 128" "C4 u_dot_v 256" "C3 u_dot_v 128" "C4 u_dot_v_sum 128"; do
  set -- $a
  for S in TE_G2_T4 TE_G8_T4 SV_G16 SV_G32 SV_G64 SV_G128 SV_G512; do
    timeout 300 python scripts/prof_op.py --config $1 --op $2 --F $3 --schedule $S --reps 20
  done
done
