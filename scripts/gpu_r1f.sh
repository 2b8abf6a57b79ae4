# usage: bash scripts/gpu_r1f.sh TAG -- power probe of C5 schedules, full sweep + corpus
T=${1:-x}
make -j8 > /dev/null 2>&1
bash scripts/gpu_power.sh
timeout 3000 python scripts/sweep.py --configs C1 C2 C3 C4 C5 --out gpurun_out/sweep_full_$T.jsonl --table gpurun_out/selector_table_$T.json 2>&1 | grep -v Warn | tail -40
timeout 1500 python scripts/selector_corpus.py --graphs 60 --budget-s 1200 --out gpurun_out/selector_corpus_$T.jsonl > gpurun_out/corpus_$T.log 2>&1
tail -2 gpurun_out/corpus_$T.log
