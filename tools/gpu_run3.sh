mkdir -p gpurun_out
timeout 300 python tools/exp_options.py --sweeps 3 --set "sampler=2" > gpurun_out/exp3.log 2>&1; cat gpurun_out/exp3.log
timeout 600 ncu --set full --clock-control none --import-source on -k 'regex:sweep_tile_kernel' -s 3 -c 1 \
    -o gpurun_out/prof_tile1 -f python tools/exp_options.py --sweeps 1 --warmup 3 --set "sampler=2" > gpurun_out/prof_tile1.log 2>&1
tail -3 gpurun_out/prof_tile1.log
