# round 2 (r2h): edge-lanes vertex kernel with a transposed butterfly and P lanes per row
# (TV_G1_T{8,16}_E1; C1 / C2 latency) and column-index prefetch in k_dott (C5 u_dot_v)
T=${1:-r2h}
EL="WV_G1_T1_E1,TV_G1_T16_E1,TV_G1_T8_E1"
CASES="C1:u_mul_e_sum:16:$EL C1:copy_u_sum:16:$EL C1:copy_u_max:16:$EL C2:copy_e_max:8:$EL,SV_G16_F8 C2:copy_u_max:8:$EL C2:copy_e_sum:8:WE_G4_T1,$EL C2:u_mul_e_sum:16:$EL C2:copy_u_sum:8:WE_G4_T1,$EL C5:u_dot_v:602:SV_G256_F128,SV_G512_F128 C3:u_dot_v:128:SV_G256_F128 C5:copy_u_sum:602:SV_G512_F128_P1"
python scripts/probe_latency.py --config C1 --schedules WV_G1_T1_E1 2>&1 | tail -3
AB_REPS=100 bash scripts/gpu_ab.sh $T "$CASES" default "" dottpf "-DUG_DOTT_PF=1"
timeout 900 python -m pytest tests/test_gpu_edgelanes.py tests/test_gpu_dott.py -x -q 2>&1 | tail -2
touch paper_conf_asplos_0001lslwlgslllw23_b200/csrc/k_dott.cu; make -j16 EXTRA="-DUG_DOTT_PF=1" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_dott.py -x -q 2>&1 | tail -2
touch paper_conf_asplos_0001lslwlgslllw23_b200/csrc/k_dott.cu; make -j16 > /dev/null 2>&1
