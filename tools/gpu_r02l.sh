LDA_TIMING=1 timeout 600 python tools/exp_options.py --config pubmed --sweeps 1 --warmup 1 > gpurun_out/r02l_loadtiming.log 2>&1
timeout 900 python bench.py --steps 20 --warmup 3 > gpurun_out/r02l_bench.json 2> gpurun_out/r02l_bench.err
bash tools/run_sanitize.sh r02l
grep "\[lda\]" gpurun_out/r02l_loadtiming.log
