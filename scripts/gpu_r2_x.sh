T=${1:-r2x}
timeout 900 python -m pytest tests/test_gpu_edgelanes.py -x -q 2>&1 | tail -2
python scripts/ab_sched.py --reps 20 --tag $T --cases "C1:u_mul_e_sum:16:TE_G1_T4,WV_G1_T1_E1" "C1:copy_u_sum:16:TE_G1_T4,WV_G1_T1_E1" "C1:copy_u_max:16:WV_G1_T1_E1" "C2:copy_u_max:8:SV_G16_F16,WV_G1_T1_E1" "C2:copy_u_sum:8:WE_G4_T1,WV_G1_T1_E1" 2>&1
timeout 1500 python scripts/sweep.py --configs C1 C2 --out gpurun_out/sweep_$T.jsonl --table gpurun_out/selector_table_$T.json 2>&1 | grep -v Warn | tail -16
