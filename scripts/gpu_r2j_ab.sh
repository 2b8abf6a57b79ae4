# round 2 (r2j): k_dott full-tile loop without the mask selects (UG_DOTT_FULL) and 32-bit gather
# offsets (UG_DOTT_O32) -- C5 u_dot_v / u_dot_v_sum, C3 / C4 wide-head SDDMM
T=${1:-r2j}
D="C5:u_dot_v:602:SV_G256_F128,SV_G512_F128 C5:u_dot_v_sum:602:SV_G512_F128,SV_G2048_F128 C3:u_dot_v:128:SV_G256_F128 C4:u_dot_v:256:SV_G128_F128,SV_G128 C4:u_dot_v:128:SV_G64,SV_G64_F128 C5:copy_u_sum:602:SV_G512_F128_P1"
AB_REPS=20 bash scripts/gpu_ab.sh $T "$D" old "-DUG_DOTT_FULL=0 -DUG_DOTT_O32=0" full "-DUG_DOTT_O32=0" full_o32 ""
timeout 900 python -m pytest tests/test_gpu_dott.py tests/test_gpu_configs.py -x -q -k "dot or dott" 2>&1 | tail -2
