set -x
make -j8 > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_api.py -x -q 2>&1 | tail -15
for S in TE_G32_T16 TE_G8_T16 WV_G8_T1 SV_G128_F128; do python scripts/prof_op.py --config C3 --op u_mul_e_sum --F 128 --schedule $S; done
python scripts/prof_op.py --config C3 --op copy_u_sum --F 128 --schedule TE_G32_T16
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_edge -s 2 -c 1 -o gpurun_out/prof_k_edge_mul_r1 python scripts/prof_op.py --config C3 --op u_mul_e_sum --F 128 --schedule TE_G32_T16 --reps 3 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_edge -s 2 -c 1 -o gpurun_out/prof_k_edge_copy_r1 python scripts/prof_op.py --config C3 --op copy_u_sum --F 128 --schedule TE_G32_T16 --reps 3 > /dev/null 2>&1
