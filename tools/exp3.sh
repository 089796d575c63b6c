python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests4.log 2>&1; tail -5 gpurun_out/gpu_tests4.log
python tools/exp_options.py --sweeps 5 --set "sampler=0" --set "sampler=1" > gpurun_out/exp4.log 2>&1; cat gpurun_out/exp4.log
LDA_LIBRARY=$PWD/variants/q2.so python tools/exp_options.py --sweeps 5 --set "sampler=1" 2>&1 | sed 's/^/q2 /'
ncu --set full --clock-control none --import-source on -k 'regex:sweep_quad_kernel' -s 3 -c 1 \
    -o gpurun_out/prof_q3 -f python tools/exp_options.py --sweeps 1 --warmup 3 --set "sampler=1" > gpurun_out/prof_q3.log 2>&1
ls gpurun_out
