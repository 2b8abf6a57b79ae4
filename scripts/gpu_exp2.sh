set -x
make -j8 > /dev/null 2>&1
for S in SV_G512_F64 SV_G512_F64_V2; do python scripts/prof_op.py --config C5 --op copy_u_sum --F 602 --schedule $S --reps 5; done
for S in SV_G512_F64 SV_G512_F128 SV_G512_F32 SV_G512_F64_V2; do python scripts/prof_op.py --config C5 --op copy_u_sum --F 602 --ld 608 --schedule $S --reps 5; done
for S in SV_G512_F64 SV_G512_F128; do python scripts/prof_op.py --config C5 --op copy_u_sum --F 602 --ld 604 --schedule $S --reps 5; done
for S in SV_G512_F64 SV_G512_F128; do
  timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sector_hit_rate.pct,l1tex__m_xbar2l1tex_read_bytes.sum,smsp__inst_executed.sum --clock-control none -k k_split -s 2 -c 1 python scripts/prof_op.py --config C5 --op copy_u_sum --F 602 --ld 608 --schedule $S --reps 3 2>&1 | grep -E "gpu__time|dram__bytes|hit_rate|xbar|inst_exec" | sed "s/^/$S /"
done
