# round 2: ncu --set full of the register SV kernel vs the staged SV kernels (C3 F = 128)
T=${1:-r2d}
for a in "copy_u_sum SV_G128_F128 k_split" "u_mul_e_sum SV_G128_F128 k_split" "copy_u_sum SV_G128_F128_A1 k_svg" \
         "copy_u_sum SV_G128_F128_M1 k_svg" "u_mul_e_sum SV_G128_F128_A1 k_svg"; do
  set -- $a
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$3 -s 2 -c 1 \
    -o gpurun_out/ncu_${T}_$1_$2 python scripts/prof_op.py --config C3 --op $1 --F 128 --schedule $2 --reps 3 \
    > gpurun_out/ncu_${T}_$1_$2.log 2>&1
  tail -1 gpurun_out/ncu_${T}_$1_$2.log
done
ls gpurun_out/*.ncu-rep
