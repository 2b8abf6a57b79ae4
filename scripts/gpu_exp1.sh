set -x
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-secondary"
$B | python -c "import json,sys; l=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('UF8', l['ms_per_step'], l['value'])"
UG_LIBRARY=build_uf16/libugraph.so $B | python -c "import json,sys; l=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('UF16', l['ms_per_step'], l['value'])"
for S in SV_G1024_F64 SV_G1024_F32 SV_G1024_F16; do
  timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sector_hit_rate.pct,lts__t_sectors_srcunit_tex_op_read.sum --clock-control none -k k_split -s 3 -c 1 $B --steps 1 --schedule $S 2>&1 | grep -E "gpu__time|dram__bytes|hit_rate|sectors_src" | sed "s/^/$S /"
done
