set -x
make -j8 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k k_split -s 1 -c 1 -o gpurun_out/prof_split_mul_r1 python scripts/prof_op.py --config C5 --op u_mul_e_sum --F 602 --schedule SV_G128_F64_P1 --reps 2 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k k_split -s 1 -c 1 -o gpurun_out/prof_split_copy_p1_r1 python scripts/prof_op.py --config C5 --op copy_u_sum --F 602 --schedule SV_G128_F64_P1 --reps 2 > /dev/null 2>&1
ls -la gpurun_out/*.ncu-rep
