mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "k_variants or edge or tile_sampler or appendix or tiny_config_lockstep or k8192" > gpurun_out/gpu_tests8.log 2>&1; tail -3 gpurun_out/gpu_tests8.log
timeout 600 python tools/exp_options.py --sweeps 5 --set "sampler=2" --set "sampler=2,tile_tokens=32000000" --set "sampler=2,tail_per_tile=128" > gpurun_out/exp8.log 2>&1; cat gpurun_out/exp8.log
timeout 600 ncu --set full --clock-control none --import-source on -k 'regex:sweep_tile_kernel' -s 3 -c 1 \
    -o gpurun_out/prof_tile6 -f python tools/exp_options.py --sweeps 1 --warmup 3 --set "sampler=2" > gpurun_out/prof_tile6.log 2>&1
tail -1 gpurun_out/prof_tile6.log
