make -j8 > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_arg.py tests/test_gpu_gat.py tests/test_gpu_api.py tests/test_gpu_autograd.py -x -q 2>&1 | tail -15
