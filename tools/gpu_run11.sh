mkdir -p gpurun_out
timeout 900 python tools/exp_options.py --sweeps 5 --set "sampler=2" --set "tile_tokens=12000000" --set "tile_tokens=24000000" --set "tail_per_tile=32" --set "tail_per_tile=96" --set "chunk_tokens=2048" --set "chunk_tokens=8192" --set "tile_tokens=12000000,tail_per_tile=96" 2>&1 | grep -v "^#"
