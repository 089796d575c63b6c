# tile size / tail threshold / chunk size sweep at PubMed shape (library defaults otherwise)
OUT=gpurun_out; mkdir -p $OUT
timeout 1500 python tools/exp_options.py --config pubmed --sweeps 10 --warmup 20 \
  --set "" --set tile_tokens=7000000 --set tile_tokens=10000000 --set tile_tokens=20000000 \
  --set tail_per_tile=32 --set tail_per_tile=128 --set chunk_tokens=2048 --set chunk_tokens=8192 --set "" 2>&1 | tee $OUT/r02ah_tiles.log
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -p no:cacheprovider -k "radix or appendix or midsize or sparse" > $OUT/r02ah_pytest.log 2>&1; echo "pytest exit $?" >> $OUT/r02ah_pytest.log; tail -2 $OUT/r02ah_pytest.log
