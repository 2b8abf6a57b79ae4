T=${1:-r2j}
./scripts/probes/minmax_zero
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "message_creation_sv_fast_path" 2>&1 | grep -E "Error|assert|passed|failed" | head -20
timeout 900 python -m pytest tests/test_gpu_nan.py -x -q 2>&1 | tail -15
timeout 900 python scripts/ab_sched.py --tag $T --cases "C3:copy_u_max:128:SV_G128_F64,SV_G128_F32" "C3:copy_u_max:32:SV_G128_F32" "C5:u_dot_v:602:SV_G512_F64,SV_G512_F128" 2>&1
