# round 2 (r2m): SV column tiles of a non-power-of-two lane count (idle lanes past ftile / vec):
# slab size vs L2 (C5: 128 cols = 119 MB of a 126 MB L2) -- parity first, then the A/B
T=${1:-r2m}
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -k "non_power" 2>&1 | tail -2
timeout 1200 python -m pytest tests/test_gpu_configs.py -x -q -k "C5_headline or C5_padded" 2>&1 | tail -2
C="C5:copy_u_sum:602:SV_G512_F128_P1,SV_G512_F120_P1,SV_G512_F112_P1,SV_G512_F96_P1,SV_G512_F128_P1 C5:u_mul_e_sum:602:SV_G2048_F128_P1,SV_G2048_F120_P1,SV_G2048_F112_P1 C3:copy_u_sum:128:SV_G128_F32,SV_G128_F24,SV_G128_F48 C3:u_mul_e_sum:128:SV_G128_F32,SV_G128_F24,SV_G128_F48 C4:copy_u_sum:128:SV_G128_F128,SV_G128_F96"
timeout 1200 python scripts/ab_sched.py --tag $T --reps 20 --cases $C 2>&1 | grep '^{'
