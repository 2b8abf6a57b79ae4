# A/B of build variants on one B200 (run under gpurun):
#   bash scripts/gpu_ab.sh TAG 'CASES' name1 '-DFLAG=1 ...' [name2 '...' ...]
# CASES as scripts/ab_sched.py --cases ("C3:u_mul_e_sum:128:SV_G128_F32,SV_G128_F64 ...").
# Each variant rebuilds libugraph.so with `make EXTRA=<flags>`, then prints one JSON line per
# (case, schedule) with the CUDA-event median; the default build is restored at the end.
# Past runs (the flags behind every profiles/r*/ab_* file): scripts/AB_HISTORY.md.
T=$1; CASES=$2; shift 2
CS=paper_conf_asplos_0001lslwlgslllw23_b200/csrc
while [ $# -ge 2 ]; do
  NAME=$1; FLAGS=$2; shift 2
  touch $CS/*.cu; make -j16 EXTRA="$FLAGS" > gpurun_out/ab_build_$T-$NAME.log 2>&1 || { echo "build $NAME failed"; tail -5 gpurun_out/ab_build_$T-$NAME.log; continue; }
  echo "== $NAME ($FLAGS)"
  timeout 900 python scripts/ab_sched.py --tag $T-$NAME --reps ${AB_REPS:-20} --cases $CASES 2>&1 | grep '^{'
done
touch $CS/*.cu; make -j16 > /dev/null 2>&1
