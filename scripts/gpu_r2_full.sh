# round 2: full GPU suite, smoke, bench (+ reference arm), launch list + ncu of the bench kernel,
# per-op ncu (C1-C4), sanitizers on the fused kernels
T=${1:-r2h}
nvidia-smi --query-gpu=name,power.limit,enforced.power.limit,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 2400 python -m pytest tests/ -m gpu -x -q 2>&1 | tail -4
timeout 900 python bench.py > gpurun_out/bench_$T.log 2>&1; tail -c 400 gpurun_out/bench_$T.log
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref_$T.log 2>&1; tail -c 300 gpurun_out/bench_ref_$T.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/launches_$T.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-secondary > /dev/null 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_split -s 3 -c 1 -o gpurun_out/prof_k_split_$T python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-secondary > gpurun_out/ncu_$T.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,lts__t_sectors_srcunit_tex_op_read.sum --clock-control none -k regex:'^k_' --csv --log-file gpurun_out/ncu_per_op_$T.csv python scripts/ncu_per_op.py run gpurun_out/ncu_per_op_order_$T.json > gpurun_out/ncu_per_op_$T.log 2>&1; tail -2 gpurun_out/ncu_per_op_$T.log
