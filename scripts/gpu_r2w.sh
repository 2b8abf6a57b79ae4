# round 2 (r2w): dot-attention packed-heads kernel, float / float2 slices at 5 CTAs / SM
T=${1:-r2w}
CS=paper_conf_asplos_0001lslwlgslllw23_b200/csrc
for v in "m4:" "m5:-DUG_DAH_MINB_NARROW=5"; do
  n=${v%%:*}; fl=${v#*:}
  touch $CS/k_dotattn.cu; make -j16 EXTRA="$fl" > /dev/null 2>&1 || { echo "build $n failed"; continue; }
  echo "== $n ($fl)"
  timeout 600 python scripts/dotattn_probe.py --tag $T-$n 2>&1 | grep '^{'
  timeout 600 python -m pytest tests/test_gpu_dotattn.py -x -q 2>&1 | tail -1
done
touch $CS/k_dotattn.cu; make -j16 > /dev/null 2>&1
