#!/bin/bash
# Round-2 profiling recipe (one GPU, under gpurun).  Usage: tools/ncu_r02.sh <tag> [config] [kernels-regex]
# 1) launch list of the bench command (our kernels; cold-cache, serialised)
# 2) one `ncu --set full --import-source on` capture of each sweep kernel
set -u
TAG=${1:-r02}
CFG=${2:-pubmed}
OUT=gpurun_out
mkdir -p $OUT
KRE='regex:^(tok_row_kernel|init_tile_kernel|sweep_tile_cta_kernel|sweep_kernel|sweep_tile_kernel|word_table_kernel|recount_kernel|theta_kernel|gather_z_kernel|prologue_kernel|zero_rows_kernel|init_kernel|ll_word_kernel|ll_doc_kernel|ll_final_kernel|peer_rs_kernel|peer_copy_kernel)'
ncu --metrics gpu__time_duration.sum --clock-control none -k "$KRE" --csv \
    --log-file $OUT/launches_${TAG}_${CFG}.csv \
    python bench.py --config $CFG --steps 2 --warmup 3 --no-cpu-baseline > $OUT/launches_${TAG}_${CFG}.bench.log 2>&1
PK=${3:-'regex:^(sweep_tile_kernel|sweep_tile_cta_kernel|word_table_kernel|recount_kernel|theta_kernel|gather_z_kernel)'}
ncu --set full --clock-control none --import-source on -k "$PK" -s 12 -c 5 \
    -o $OUT/prof_${TAG}_${CFG} -f \
    python bench.py --config $CFG --steps 1 --warmup 3 --no-cpu-baseline > $OUT/prof_${TAG}_${CFG}.log 2>&1
ls -la $OUT | tail -5
