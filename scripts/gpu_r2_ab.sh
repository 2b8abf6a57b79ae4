T=${1:-r2ab}
timeout 900 python -m pytest tests/test_gpu_edgelanes.py -x -q 2>&1 | tail -2
python scripts/ab_sched.py --tag $T --cases "C5:u_add_v:1:WE_G4_T1,SV_G1024_E1,SV_G4096_E1" "C2:u_add_v:8:TE_G1_T1,SV_G64_E1" "C4:u_add_v:128:SV_G64_F64" 2>&1
