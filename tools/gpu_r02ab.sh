OUT=gpurun_out; mkdir -p $OUT
LDA_TIMING=1 python tools/load_only.py --config pubmed --reps 3 --pinned > $OUT/r02ab_load_pinned.log 2>&1
grep -E "sorter|copiers|load [0-9]|layout done|H2D|init" $OUT/r02ab_load_pinned.log
LDA_TIMING=1 python tools/load_only.py --config pubmed --reps 2 > $OUT/r02ab_load.log 2>&1
grep -E "sorter|copiers|load [0-9]|layout done" $OUT/r02ab_load.log
timeout 900 python tools/exp_options.py --config pubmed --sweeps 10 --warmup 20 2>&1 | tail -1
