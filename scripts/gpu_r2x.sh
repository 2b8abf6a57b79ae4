# round 2 (r2x): parity of the contiguous edge-weight modes (BM 6 / 7, merge instance) on a large sparse graph
timeout 1500 python -m pytest tests/test_gpu_bm67.py -x -q 2>&1 | tail -3
