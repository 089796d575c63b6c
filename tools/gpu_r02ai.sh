OUT=gpurun_out; mkdir -p $OUT
timeout 1500 python tools/exp_options.py --config pubmed --sweeps 10 --warmup 20 \
  --set "" --set tail_per_tile=32,chunk_tokens=2048 --set tail_per_tile=16 --set tail_per_tile=16,chunk_tokens=2048 \
  --set chunk_tokens=1024 --set tail_per_tile=32,chunk_tokens=1024 --set tail_per_tile=32,chunk_tokens=2048,tile_tokens=10000000 \
  --set tail_per_tile=24,chunk_tokens=1536 --set "" 2>&1 | tee $OUT/r02ai_tiles.log
for c in nytimes nytimes_k128; do
timeout 900 python tools/exp_options.py --config $c --sweeps 10 --warmup 20 --set "" --set tail_per_tile=32,chunk_tokens=2048 --set tail_per_tile=16,chunk_tokens=2048 --set "" 2>&1 | tee -a $OUT/r02ai_tiles.log
done
