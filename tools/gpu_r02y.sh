# A/B: packed fp32 walk (F32X2) on / off at PubMed + K = 8192; sparse rows on / off with the prefetching table kernel
OUT=gpurun_out; mkdir -p $OUT
timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -p no:cacheprovider -k "8192 or sparse or k_variants or tile_sampler or tiny" > $OUT/r02y_pytest.log 2>&1; echo "pytest exit $?" >> $OUT/r02y_pytest.log
tail -2 $OUT/r02y_pytest.log
bash tools/gpu_variants.sh r02y pubmed f2on nof2
bash tools/gpu_variants.sh r02y8 nytimes_k8192 f2on nof2
timeout 900 python tools/exp_options.py --config nytimes_k8192 --sweeps 10 --warmup 20 --set sparse_words=0 --set sparse_words=-1 --set sparse_words=0 --set sparse_words=-1 2>&1 | tee $OUT/r02y_sparse.log
