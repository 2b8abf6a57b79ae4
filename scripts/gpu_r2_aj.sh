# round 2: k_gat register budget / L2 hints A/B (r2aj-r2al); the final form picks 6 CTAs/SM for
# float4 slices of large grids (r2am checks it against the fixed budgets)
T=${1:-r2am}
timeout 600 python scripts/dotattn_probe.py --gat --tag $T 2>&1
timeout 900 python -m pytest tests/test_gpu_gat.py -x -q 2>&1 | tail -2
