T=${1:-r2k}
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_nan.py tests/test_gpu_dott.py -x -q 2>&1 | tail -3
timeout 900 python scripts/ab_sched.py --tag $T --cases "C3:copy_u_max:128:SV_G128_F64" "C3:copy_u_max:32:SV_G128_F32" \
  "C5:u_dot_v:602:SV_G512_F32,SV_G512_F64,SV_G512_F128,SV_G2048_F64" "C4:u_dot_v:256:SV_G64,SV_G256_F64,SV_G256_F128" 2>&1
