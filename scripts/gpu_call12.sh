set -x
make -j8 > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_api.py -x -q 2>&1 | tail -4
timeout 900 python -m pytest tests/test_gpu_configs.py -x -q -k "C5_headline or C5_padded" 2>&1 | tail -3
for S in SV_G512_F64 SV_G512_F64_P1 SV_G512_F128_P1 SV_G128_F64_P1 SV_G2048_F64_P1; do python scripts/prof_op.py --config C5 --op copy_u_sum --F 602 --schedule $S --reps 5; done
for S in SV_G128_F32 SV_G512_F64_P1 SV_G128_F64_P1; do python scripts/prof_op.py --config C5 --op u_mul_e_sum --F 602 --schedule $S --reps 3; done
for S in SV_G512_F64_P1 SV_G512_F128_P1; do python scripts/prof_op.py --config C5 --op copy_u_max --F 602 --schedule $S --reps 3; done
