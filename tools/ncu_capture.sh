#!/bin/bash
# Profiling recipe (run under gpurun; one GPU).  Usage:
#   tools/ncu_capture.sh <tag> [config]
# 1) launch list of the bench command (device time per launch, our kernels only)
# 2) one `ncu --set full` capture of each kernel of a sweep
set -u
TAG=${1:-r01}
CFG=${2:-pubmed}
OUT=gpurun_out
mkdir -p $OUT
KRE='regex:^(tok_row_kernel|init_tile_kernel|sweep_tile_cta_kernel|sweep_kernel|sweep_quad_kernel|sweep_tile_kernel|word_table_kernel|recount_kernel|theta_kernel|gather_z_kernel|prologue_kernel|zero_rows_kernel|init_kernel|ll_word_kernel|ll_doc_kernel|ll_final_kernel)'
ncu --metrics gpu__time_duration.sum --clock-control none -k "$KRE" --csv \
    --log-file $OUT/launches_${TAG}_${CFG}.csv \
    python bench.py --config $CFG --steps 2 --warmup 3 --no-cpu-baseline > $OUT/launches_${TAG}_${CFG}.bench.log 2>&1
ncu --set full --clock-control none --import-source on \
    -k 'regex:^(sweep_tile_kernel|word_table_kernel|recount_kernel|theta_kernel|gather_z_kernel|prologue_kernel)' -s 12 -c 6 \
    -o $OUT/prof_${TAG}_${CFG} -f \
    python bench.py --config $CFG --steps 1 --warmup 3 --no-cpu-baseline > $OUT/prof_${TAG}_${CFG}.log 2>&1
ls -la $OUT
