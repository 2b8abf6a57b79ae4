T=${1:-r2z}
timeout 900 python -m pytest tests/test_gpu_views_r2.py -x -q 2>&1 | tail -3
timeout 900 compute-sanitizer --tool memcheck python scripts/sanitize.py > gpurun_out/sanitize_memcheck_$T.log 2>&1; tail -2 gpurun_out/sanitize_memcheck_$T.log
timeout 900 compute-sanitizer --tool racecheck python scripts/sanitize.py > gpurun_out/sanitize_racecheck_$T.log 2>&1; tail -2 gpurun_out/sanitize_racecheck_$T.log
