make -j8 > /dev/null 2>&1
cd scripts
for F in 32 128; do
python time_ops.py C3 u_mul_e_sum $F SV_G128_F$F SV_G512_F$F SV_G32_F$F
python time_ops.py C3 copy_u_sum $F SV_G128_F$F SV_G32_F$F
done
python time_ops.py C1 u_mul_e_sum 16 SV_G16_F16 SV_G32_F16 SV_G128_F16 SV_G16_F64
python time_ops.py C2 u_mul_e_sum 64 SV_G16_F64 SV_G32_F64 SV_G128_F64
python time_ops.py C5 copy_u_sum 602 SV_G512_F128_P1
cd ..; timeout 900 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -2
