# round 2 evidence run: smoke, full GPU suite, bench + reference arm, launch list + ncu of the bench
# kernel, per-op ncu (C1-C4), ncu --set full of the kernels changed in round 2's second session
# (k_split BM 7 on C3 u_mul_e_sum, k_dott on C5 u_dot_v, k_vertex_el on C2 copy_e_max), N=2 gloo
# dry run, sweep with the shipped selector (Fig. 12, + a table from it), the sanitizer driver (plain)
T=${1:-r2final}
nvidia-smi --query-gpu=name,power.limit,enforced.power.limit,clocks.max.sm --format=csv
EL="TV_G1_T16_E1,TV_G1_T8_E1,WV_G1_T1_E1"
AB_REPS=200 bash scripts/gpu_ab.sh $T "C2:copy_e_max:8:$EL C2:copy_u_max:8:$EL C2:copy_u_sum:8:$EL C1:copy_u_sum:8:$EL C2:u_mul_e_sum:8:$EL" elcap6 "" elnocap "-DUG_EL_MINB_NARROW=1" > gpurun_out/ab_el_$T.jsonl 2>&1
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 2400 python -m pytest tests/ -m gpu -q 2>&1 | tail -4
timeout 900 python bench.py > gpurun_out/bench_$T.log 2>&1; tail -c 300 gpurun_out/bench_$T.log
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref_$T.log 2>&1; tail -c 200 gpurun_out/bench_ref_$T.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/launches_$T.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-secondary > /dev/null 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:'^k_split$' -s 3 -c 1 -o gpurun_out/prof_k_split_$T python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-secondary > gpurun_out/ncu_$T.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,lts__t_sectors_srcunit_tex_op_read.sum --clock-control none -k regex:'^k_' --csv --log-file gpurun_out/ncu_per_op_$T.csv python scripts/ncu_per_op.py run gpurun_out/ncu_per_op_order_$T.json > gpurun_out/ncu_per_op_$T.log 2>&1; tail -1 gpurun_out/ncu_per_op_$T.log
for c in "C3:u_mul_e_sum:128:SV_G128_F32:k_split" "C5:u_dot_v:602:SV_G256_F128:k_dott" "C2:copy_e_max:8:TV_G1_T16_E1:k_vertex_el"; do
  IFS=: read cfg op F sch k <<< "$c"
  timeout 900 ncu --set full --clock-control none -k regex:"^$k\$" -s 2 -c 1 -o /tmp/prof_${cfg}_${op}_$T python scripts/ab_sched.py --tag x --reps 2 --cases $cfg:$op:$F:$sch > /dev/null 2>&1
  # summarised here, report left in /tmp: gpurun_out must stay under 64 MiB to come back
  python scripts/ncu_summary.py full /tmp/prof_${cfg}_${op}_$T.ncu-rep > gpurun_out/prof_${cfg}_${op}_$T.json 2>&1
done
UG_DIST_BACKEND=gloo timeout 1200 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 5 --warmup 3 > gpurun_out/bench_dry2_$T.log 2>&1; tail -c 300 gpurun_out/bench_dry2_$T.log
timeout 2400 python scripts/sweep.py --configs C1 C2 C3 C4 C5 --reps 10 --out gpurun_out/sweep_$T.jsonl --table gpurun_out/selector_table_$T.json 2>&1 | grep -v Warn | tail -3
# compute-sanitizer is closed on the GPU pool since the r2fa run (profiles/sanitizer/r2_*.log are
# the last clean runs); the driver itself still runs every kernel family once, bounds-checked by
# the binding and compared with nothing -- a crash / illegal address still fails it
timeout 600 python scripts/sanitize.py 2>&1 | tail -1
du -sh gpurun_out/* | sort -h | tail -5
