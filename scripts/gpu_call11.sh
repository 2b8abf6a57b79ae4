set -x
make -j8 > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_api.py -x -q 2>&1 | tail -4
timeout 900 compute-sanitizer --tool memcheck --error-exitcode 9 python scripts/sanitize.py 2>&1 | tail -2
timeout 900 compute-sanitizer --tool racecheck --error-exitcode 9 python scripts/sanitize.py 2>&1 | tail -2
for S in SV_G512 SV_G2048 BE_G256 TE_G2_T32; do python scripts/prof_op.py --config C5 --op u_dot_v --F 602 --schedule $S --reps 3; done
for S in SV_G512 WE_G128_T1; do python scripts/prof_op.py --config C5 --op u_dot_v_sum --F 602 --schedule $S --reps 3; done
for S in SV_G512 SV_G128 TE_G2_T4; do python scripts/prof_op.py --config C4 --op u_dot_v --F 256 --schedule $S; python scripts/prof_op.py --config C4 --op u_dot_v --F 128 --schedule $S; done
for S in TE_G32_T16 TE_G32_T16_F64 TE_G32_T8_F32 TE_G8_T8_F32 SV_G128_F128; do python scripts/prof_op.py --config C3 --op copy_u_sum --F 128 --schedule $S; python scripts/prof_op.py --config C3 --op u_mul_e_sum --F 128 --schedule $S; done
timeout 1200 python -m pytest tests/test_gpu_configs.py -x -q -k "C4 or C5_headline" 2>&1 | tail -3
