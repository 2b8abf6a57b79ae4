# round 2: ncu --set full of the kernels beside the headline (one launch each, after warm-up)
T=${1:-r2ac}
run() { timeout 900 ncu --set full --clock-control none --import-source on -k regex:"$1" -s 2 -c 1 -o gpurun_out/ncu_${T}_$2 "${@:3}" > gpurun_out/ncu_${T}_$2.log 2>&1; tail -1 gpurun_out/ncu_${T}_$2.log; }
run '^k_dotsv$' dotsv_C4 python scripts/prof_op.py --config C4 --op u_dot_v --F 128 --reps 3
run '^k_dott$' dott_C5 python scripts/prof_op.py --config C5 --op u_dot_v --F 602 --schedule SV_G256_F128 --reps 3
run '^k_gat' gat_C2 python scripts/prof_fused.py --config C2 --kind gat --H 8 --F 64
run '^k_dotattn' dotattn_C4 python scripts/prof_fused.py --config C4 --kind dot --H 8 --F 128
run '^k_msg_el' msgel_C5 python scripts/prof_op.py --config C5 --op u_add_v --F 1 --schedule SV_G4096_E1 --reps 3
run '^k_split$' split_C3_mul python scripts/prof_op.py --config C3 --op u_mul_e_sum --F 128 --schedule SV_G128_F32 --reps 3
run '^k_split$' split_C3_copy python scripts/prof_op.py --config C3 --op copy_u_sum --F 128 --schedule SV_G128_F32 --reps 3
ls gpurun_out/ncu_${T}_*.ncu-rep
