# round 2 (r2k): full GPU suite + bench on the tree with BM 6 / 7, the k_dott full-tile loop and
# the edge-lanes TV schedules
T=${1:-r2k}
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 2400 python -m pytest tests/ -m gpu -q 2>&1 | tail -4
timeout 900 python bench.py > gpurun_out/bench_$T.log 2>&1; tail -c 300 gpurun_out/bench_$T.log
