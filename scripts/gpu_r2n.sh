# round 2 (r2n): segmented edge lanes (WV_Gg_T1_E1, g rows sharing a warp's lanes) -- parity,
# then C1 / C2 latency against the TV / WV edge-lanes schedules
T=${1:-r2n}
timeout 1200 python -m pytest tests/test_gpu_edgelanes.py tests/test_gpu_parity.py -x -q -k "edgelanes or non_power" 2>&1 | tail -2
EL="WV_G1_T1_E1,TV_G1_T16_E1,TV_G1_T8_E1,WV_G2_T1_E1,WV_G4_T1_E1,WV_G8_T1_E1"
C="C1:u_mul_e_sum:16:$EL C1:copy_u_sum:16:$EL C1:copy_u_max:16:$EL C2:copy_e_max:8:$EL C2:copy_u_max:8:$EL C2:copy_e_sum:8:$EL C2:copy_u_sum:8:$EL C1:copy_u_sum:8:$EL"
timeout 1200 python scripts/ab_sched.py --tag $T --reps 200 --cases $C 2>&1 | grep '^{'
