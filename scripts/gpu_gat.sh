# usage: bash scripts/gpu_gat.sh -- GAT fused-traversal parity + timing across chunk sizes
make -j8 > /dev/null 2>&1
timeout 400 python -m pytest tests/test_gpu_gat.py -x -q 2>&1 | tail -5
cd scripts
for G in 16 32 64 128; do echo "G=$G"; UG_GAT_CHUNK=$G timeout 200 python gat_probe.py 2>/dev/null; done
