# round 2 (r2u): SV message creation with the store form unswitched (UG_ASSIGN_UNSWITCH)
T=${1:-r2u}
C="C4:u_add_v:128:SV_G64_F64,SV_G64_F128 C3:u_add_v:32:SV_G64_F32 C2:u_add_v:64:SV_G16_F64 C4:u_add_v:256:SV_G64_F64"
AB_REPS=30 bash scripts/gpu_ab.sh $T "$C" fused "-DUG_ASSIGN_UNSWITCH=0" unswitched ""
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edgelanes.py -x -q -k "message_creation" 2>&1 | tail -1
