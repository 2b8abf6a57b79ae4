set -x
make -j8 > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_api.py -x -q -k chunked 2>&1 | grep -E "Error|error|assert" | head -20
timeout 900 python -m pytest tests/test_gpu_configs.py -x -q -k "positive" 2>&1 | tail -5
