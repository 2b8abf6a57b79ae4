# round 2 (r2y): per-op ncu (DRAM / L2 bytes, hit rate) of the final tree's C1-C4 bench ops, and
# ncu --set full of k_dotsv message creation at its 5-CTA budget (C4 u_dot_v F = 128)
T=${1:-r2y}
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,lts__t_sectors_srcunit_tex_op_read.sum --clock-control none -k regex:'^k_' --csv --log-file gpurun_out/ncu_per_op_$T.csv python scripts/ncu_per_op.py run gpurun_out/ncu_per_op_order_$T.json > gpurun_out/ncu_per_op_$T.log 2>&1; tail -1 gpurun_out/ncu_per_op_$T.log
timeout 600 ncu --set full --clock-control none -k regex:'^k_dotsv' -s 2 -c 1 -o /tmp/prof_dotsv_$T python scripts/ab_sched.py --tag x --reps 2 --cases C4:u_dot_v:128:SV_G32 > /dev/null 2>&1
python scripts/ncu_summary.py full /tmp/prof_dotsv_$T.ncu-rep > gpurun_out/prof_C4_u_dot_v_$T.json 2>&1
head -c 600 gpurun_out/prof_C4_u_dot_v_$T.json
