python tools/qdebug.py 2>&1 | tail -4
python tools/exp_options.py --sweeps 5 --set "sampler=0" --set "sampler=1" > gpurun_out/exp5.log 2>&1; cat gpurun_out/exp5.log
python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests5.log 2>&1; tail -3 gpurun_out/gpu_tests5.log
