#!/bin/bash
# One `ncu --set full --import-source on` capture of the sampling kernel per
# bench config, at a steady-state sweep (the 23rd launch: after bench.py's
# e2e pass of 20 sweeps and 2 warm-up sweeps), plus the pubmed launch list.
# Usage (GPU box): bash tools/ncu_configs.sh <tag> cfg1 cfg2 ...
TAG=$1; shift
OUT=gpurun_out; mkdir -p $OUT
for CFG in "$@"; do
  ncu --set full --clock-control none --import-source on -k 'regex:^(sweep_tile_kernel|sweep_tile_cta_kernel|sweep_kernel)' \
      -s 22 -c 1 -o $OUT/prof_${TAG}_${CFG} -f \
      python bench.py --config $CFG --steps 20 --warmup 3 --no-cpu-baseline > $OUT/prof_${TAG}_${CFG}.log 2>&1
  python tools/write_traffic.py $OUT/prof_${TAG}_${CFG}.ncu-rep $CFG $TAG >> $OUT/traffic_${TAG}.log 2>&1
done
KRE='regex:^(tok_row_kernel|init_tile_kernel|sweep_tile_cta_kernel|sweep_kernel|sweep_tile_kernel|word_table_kernel|recount_kernel|theta_kernel|gather_z_kernel|prologue_kernel|zero_rows_kernel|init_kernel|ll_word_kernel|ll_doc_kernel|ll_final_kernel)'
ncu --metrics gpu__time_duration.sum --clock-control none -k "$KRE" --csv \
    --log-file $OUT/launches_${TAG}_pubmed.csv \
    python bench.py --config pubmed --steps 2 --warmup 3 --no-cpu-baseline > $OUT/launches_${TAG}_pubmed.bench.log 2>&1
cp profiles/traffic.json $OUT/traffic_${TAG}.json
cat $OUT/traffic_${TAG}.log
