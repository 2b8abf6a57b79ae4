# C5 copy_u_sum: L2 evict_last fraction of the X slab loads, CTA size, chunk size
T=${1:-r2y}
CASES='C5:copy_u_sum:602:SV_G512_F128_P1,SV_G512_F128_P1_B128,SV_G1024_F128_P1,SV_G256_F128_P1 C5:u_mul_e_sum:602:SV_G2048_F128_P1 C3:copy_u_sum:128:SV_G128_F32'
python scripts/ab_sched.py --tag $T-keep1.0 --cases $CASES 2>&1
for FR in 0.75 0.5; do
  touch paper_conf_asplos_0001lslwlgslllw23_b200/csrc/k_split*.cu; make -j16 EXTRA="-DUG_KEEP_FRACTION=$FR" > /dev/null 2>&1
  python scripts/ab_sched.py --tag $T-keep$FR --cases $CASES 2>&1
done
touch paper_conf_asplos_0001lslwlgslllw23_b200/csrc/k_split*.cu; make -j16 > /dev/null 2>&1
