# round 2: fused dot attention parity; ncu of k_dott on C5
T=${1:-r2g}
timeout 1200 python -m pytest tests/test_gpu_dotattn.py -x -q 2>&1 | tail -5
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${T}_dott.csv \
  python scripts/prof_op.py --config C5 --op u_dot_v --F 602 --schedule SV_G512_F128 --reps 2 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_dott -s 1 -c 1 \
  -o gpurun_out/ncu_${T}_dott_C5 python scripts/prof_op.py --config C5 --op u_dot_v --F 602 --schedule SV_G512_F128 --reps 2 \
  > gpurun_out/ncu_${T}_dott_C5.log 2>&1; tail -2 gpurun_out/ncu_${T}_dott_C5.log
