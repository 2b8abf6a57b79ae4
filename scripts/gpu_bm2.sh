# usage: bash scripts/gpu_bm2.sh -- register budget / gathers-in-flight A/B for the SV fast path
# with a per-edge scalar B operand (BM = 2: u_mul_e_sum and friends)
for V in "5 4" "6 4" "8 4" "5 8" "6 8"; do
  set -- $V
  echo "== UG_BM2_MINB=$1 UG_BM2_UF=$2"
  make -B -j16 EXTRA="-DUG_BM2_MINB=$1 -DUG_BM2_UF=$2" > gpurun_out/bm2_build_$1_$2.log 2>&1 || { tail -5 gpurun_out/bm2_build_$1_$2.log; continue; }
  grep -A2 "_ZN2ug7k_splitILi3ELi1ELi4ELi2EE" build/k_split_mul.ptxas.log | grep -o "Used [0-9]* registers.*" | head -1
  for a in "C3 128 SV_G512_F128_P1" "C3 128 SV_G128_F64" "C3 32 SV_G128_F32" "C2 64 SV_G16_F64" "C5 602 SV_G512_F128_P1"; do
    set -- $a
    timeout 300 python scripts/prof_op.py --config $1 --op u_mul_e_sum --F $2 --schedule $3 --reps 20 2>&1 | tail -1
  done
done
make -B -j16 > /dev/null 2>&1
