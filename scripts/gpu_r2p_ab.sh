# round 2 (r2p): gathers in flight of the 8-CTA contiguous-weight loop (BM 7) with the FMA fold
T=${1:-r2p}
C="C3:u_mul_e_sum:128:SV_G128_F32,SV_G128_F64 C3:u_mul_e_sum:32:SV_G128_F32 C4:u_mul_e_sum:128:SV_G128_F128 C3:copy_u_sum:128:SV_G128_F32"
AB_REPS=30 bash scripts/gpu_ab.sh $T "$C" uf4 "" uf8 "-DUG_BM7_UF=8"
