# usage: bash scripts/gpu_final2.sh TAG -- gpu_final.sh + compute-sanitizer (memcheck, racecheck, synccheck)
T=${1:-x}
set -x
make -j8 > /dev/null 2>&1
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 2400 python -m pytest tests/ -m gpu -x -q 2>&1 | tail -4
timeout 900 python bench.py > gpurun_out/bench_$T.log 2>&1; tail -c 300 gpurun_out/bench_$T.log
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref_$T.log 2>&1; tail -c 300 gpurun_out/bench_ref_$T.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/launches_$T.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-secondary > /dev/null 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k k_split -s 3 -c 1 -o gpurun_out/prof_k_split_$T python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-secondary > gpurun_out/ncu_$T.log 2>&1
grep -o '"schedule": "[A-Z0-9_]*"' gpurun_out/ncu_$T.log | head -1
for TOOL in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $TOOL python scripts/sanitize.py > gpurun_out/sanitize_${TOOL}_$T.log 2>&1
  tail -2 gpurun_out/sanitize_${TOOL}_$T.log
done
