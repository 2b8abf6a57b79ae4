# round 2 (r2o): where C2's ~4 us above an empty kernel go -- ncu of the edge-lanes kernels on C2
# copy_e_max (F = 8) and C1 u_mul_e_sum; plus a dry pass of the extended sanitizer driver
T=${1:-r2o}
python scripts/sanitize.py 2>&1 | tail -2
for c in "C2:copy_e_max:8:TV_G1_T16_E1" "C2:copy_e_max:8:WV_G4_T1_E1" "C1:u_mul_e_sum:16:WV_G1_T1_E1" "C2:copy_u_sum:64:SV_G16_F64"; do
  n=$(echo $c | tr ':' '_')
  timeout 600 ncu --set full --clock-control none -k regex:'^k_' -s 3 -c 1 -o gpurun_out/ncu_${T}_$n python scripts/ab_sched.py --tag x --reps 3 --cases $c > /dev/null 2>&1
  ncu -i gpurun_out/ncu_${T}_$n.ncu-rep --page details --csv 2>/dev/null | grep -E '"Duration"|"Elapsed Cycles"|"Achieved Occupancy"|"Registers Per Thread"|"Grid Size"|"Waves Per SM"|"Memory Throughput"|"L2 Hit Rate"' | head -12
done
