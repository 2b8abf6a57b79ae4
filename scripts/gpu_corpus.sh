# usage: bash scripts/gpu_corpus.sh TAG -- learned-selector corpus (f4) + a default bench line
T=${1:-x}
set -x
make -j8 > /dev/null 2>&1
timeout 2300 python scripts/selector_corpus.py --graphs 60 --budget-s 2100 --out gpurun_out/selector_corpus_$T.jsonl > gpurun_out/corpus_$T.log 2>&1
tail -3 gpurun_out/corpus_$T.log
timeout 900 python bench.py > gpurun_out/bench_$T.log 2>&1; tail -c 400 gpurun_out/bench_$T.log
