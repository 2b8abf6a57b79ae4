# round 2: learned-selector corpus on the round-2 kernels (60 synthetic Chung-Lu graphs x op classes x F)
T=${1:-r2q}
timeout 2700 python scripts/selector_corpus.py --graphs 60 --budget-s 2400 --out gpurun_out/selector_corpus_$T.jsonl > gpurun_out/corpus_$T.log 2>&1
tail -3 gpurun_out/corpus_$T.log; wc -l gpurun_out/selector_corpus_$T.jsonl
