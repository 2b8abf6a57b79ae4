# verification of a committed tree: smoke, full GPU suite, bench + reference arm, launch list
T=${1:-verify}
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 2400 python -m pytest tests/ -m gpu -q 2>&1 | tail -3
timeout 900 python bench.py > gpurun_out/bench_$T.log 2>&1; tail -c 200 gpurun_out/bench_$T.log
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref_$T.log 2>&1; tail -c 150 gpurun_out/bench_ref_$T.log
