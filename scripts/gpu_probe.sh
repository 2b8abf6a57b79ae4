# usage: bash scripts/gpu_probe.sh TAG -- in-bench vs isolated timing of the C5 kernel; ncu of the C3/C4 kernels
T=${1:-x}
set -x
make -j8 > /dev/null 2>&1
timeout 600 python scripts/probe_c5.py 2>&1 | tail -8
for S in SV_G32_F32 SV_G16_F32 TE_G8_T4; do timeout 300 python scripts/prof_op.py --config C3 --op copy_u_sum --F 32 --schedule $S --reps 20; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_split -s 2 -c 1 -o gpurun_out/prof_c3f32_$T python scripts/prof_op.py --config C3 --op copy_u_sum --F 32 --schedule SV_G32_F32 --reps 3 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_split -s 2 -c 1 -o gpurun_out/prof_c3f128_$T python scripts/prof_op.py --config C3 --op copy_u_sum --F 128 --schedule SV_G32_F128 --reps 3 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_ -s 2 -c 1 -o gpurun_out/prof_c4dot_$T python scripts/prof_op.py --config C4 --op u_dot_v --F 128 --schedule TE_G2_T4 --reps 3 > /dev/null 2>&1
ls gpurun_out
