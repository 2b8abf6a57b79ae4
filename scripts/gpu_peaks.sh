# FFMA and L2 -> SM read peaks (scripts/probes/peaks.cu), three runs
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/peaks scripts/probes/peaks.cu || exit 1
for i in 1 2 3; do /tmp/peaks; done > gpurun_out/peaks.jsonl
cat gpurun_out/peaks.jsonl
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm,power.draw --format=csv
