T=r2gat
CS=paper_conf_asplos_0001lslwlgslllw23_b200/csrc
for m in 0 1; do
  touch $CS/k_gat.cu; make -j16 EXTRA="-DUG_GAT_O32=$m" > /dev/null 2>&1 || { echo "build $m failed"; continue; }
  echo "== o32=$m"
  timeout 600 python scripts/dotattn_probe.py --gat --tag $T-o32$m 2>&1 | grep '^{'
  timeout 600 python -m pytest tests/test_gpu_gat.py -x -q 2>&1 | tail -1
done
touch $CS/k_gat.cu; make -j16 > /dev/null 2>&1
