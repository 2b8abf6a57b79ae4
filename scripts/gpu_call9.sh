set -x
make -j8 > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_api.py -x -q 2>&1 | tail -3
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python scripts/sanitize.py > gpurun_out/sanitize_$tool.log 2>&1; echo "$tool rc=$?"; tail -3 gpurun_out/sanitize_$tool.log
done
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_r1g.log 2>&1; tail -c 400 gpurun_out/bench_r1g.log
