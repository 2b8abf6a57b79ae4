# usage: bash scripts/gpu_resweep.sh TAG -- full sweep -> selector table, learned-selector corpus, bench line
T=${1:-x}
set -x
make -j8 > /dev/null 2>&1
timeout 3000 python scripts/sweep.py --configs C1 C2 C3 C4 C5 --out gpurun_out/sweep_full_$T.jsonl --table gpurun_out/selector_table_$T.json 2>&1 | grep -v Warn | tail -40
timeout 1500 python scripts/selector_corpus.py --graphs 60 --budget-s 1200 --out gpurun_out/selector_corpus_$T.jsonl > gpurun_out/corpus_$T.log 2>&1
tail -2 gpurun_out/corpus_$T.log
