# round 2: k_dott (SV dot with column tiles, any head width) parity + A/B; staged-SV build sweep
T=${1:-r2f}
timeout 1500 python -m pytest tests/test_gpu_dott.py -x -q 2>&1 | tail -5
timeout 900 python scripts/ab_sched.py --tag $T --cases \
  "C4:u_dot_v:128:SV_G64,SV_G64_F128,SV_G256_F128,SV_G64_F64" \
  "C4:u_dot_v:256:SV_G64,SV_G64_F128,SV_G256_F128" \
  "C4:u_dot_v_sum:128:SV_G64,SV_G64_F128,SV_G256_F128" \
  "C3:u_dot_v:128:SV_G128,SV_G64_F128,SV_G256_F128" \
  "C5:u_dot_v:602:BE_G256,SV_G512_F128,SV_G2048_F128,SV_G512_F64" \
  "C5:u_dot_v_sum:602:WE_G128_T1,SV_G512_F128" \
  "C5:copy_u_sum:602:SV_G512_F128_P1" \
  2>&1 | tee gpurun_out/ab_$T.jsonl
for V in "8 12" "8 8" "4 24" "16 6"; do
  set -- $V
  touch paper_conf_asplos_0001lslwlgslllw23_b200/csrc/k_svg_*.cu
  make -j16 EXTRA="-DUG_SVG_WARPS=$1 -DUG_SVG_RING_KB=$2" > gpurun_out/svg_build_$1_$2.log 2>&1 || { tail -3 gpurun_out/svg_build_$1_$2.log; continue; }
  timeout 600 python scripts/ab_sched.py --tag "$T-w$1-kb$2" --cases \
    "C3:copy_u_sum:128:SV_G128_F128_M1,SV_G128_F128_A1" "C3:u_mul_e_sum:128:SV_G128_F128_M1,SV_G128_F128_A1" \
    "C5:copy_u_sum:602:SV_G512_F128_P1_M1" "C5:u_mul_e_sum:602:SV_G512_F128_P1_M1" 2>&1 | tee -a gpurun_out/ab_$T.jsonl
done
touch paper_conf_asplos_0001lslwlgslllw23_b200/csrc/k_svg_*.cu; make -j16 > /dev/null 2>&1
