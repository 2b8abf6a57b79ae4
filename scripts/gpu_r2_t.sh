T=${1:-r2t}
CASES='C5:u_dot_v:602:SV_G256_F128,SV_G512_F128,SV_G2048_F128 C4:u_dot_v:128:SV_G256_F128'
python scripts/ab_sched.py --tag $T-minb6 --cases $CASES 2>&1
touch paper_conf_asplos_0001lslwlgslllw23_b200/csrc/k_dott.cu; make -j16 EXTRA="-DUG_DOTT_MINB=8" > /dev/null 2>&1
python scripts/ab_sched.py --tag $T-minb8 --cases $CASES 2>&1
touch paper_conf_asplos_0001lslwlgslllw23_b200/csrc/k_dott.cu; make -j16 > /dev/null 2>&1
python - <<'PY'
import os, statistics, torch, sys
sys.path.insert(0, '.')
import paper_conf_asplos_0001lslwlgslllw23_b200 as ug, ugdata
for cfg, H, F in (("C4", 1, 128), ("C4", 8, 128), ("C2", 8, 64)):
    c = ugdata.CONFIGS[cfg]; s, d = ugdata.graph(cfg); g = ug.Graph(c.V, s, d)
    z = torch.randn(c.V, F, device="cuda"); o = torch.empty_like(z)
    for _ in range(3): ug.dot_attention(g, z, z, z, H, out=o)
    ts = []
    for _ in range(20):
        torch.cuda._sleep(200000); e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); ug.dot_attention(g, z, z, z, H, out=o); e1.record(); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1) * 1e3)
    print(cfg, H, F, os.environ.get("UG_DOTATTN_WIDE"), round(statistics.median(ts), 1), "us")
PY
UG_DOTATTN_WIDE=1 python - <<'PY'
import os, statistics, torch, sys
sys.path.insert(0, '.')
import paper_conf_asplos_0001lslwlgslllw23_b200 as ug, ugdata
for cfg, H, F in (("C4", 1, 128), ("C4", 8, 128), ("C2", 8, 64)):
    c = ugdata.CONFIGS[cfg]; s, d = ugdata.graph(cfg); g = ug.Graph(c.V, s, d)
    z = torch.randn(c.V, F, device="cuda"); o = torch.empty_like(z)
    for _ in range(3): ug.dot_attention(g, z, z, z, H, out=o)
    ts = []
    for _ in range(20):
        torch.cuda._sleep(200000); e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); ug.dot_attention(g, z, z, z, H, out=o); e1.record(); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1) * 1e3)
    print(cfg, H, F, os.environ.get("UG_DOTATTN_WIDE"), round(statistics.median(ts), 1), "us")
PY
