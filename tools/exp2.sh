# parity tests, then timing + one ncu --set full capture of each sampler
python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests3.log 2>&1; tail -5 gpurun_out/gpu_tests3.log
python tools/exp_options.py --sweeps 5 --set "sampler=0" --set "sampler=1" > gpurun_out/exp3.log 2>&1; cat gpurun_out/exp3.log
for S in 1 0; do
ncu --set full --clock-control none --import-source on -k 'regex:sweep_(quad_)?kernel' -s 3 -c 1 \
    -o gpurun_out/prof_s$S -f python tools/exp_options.py --sweeps 1 --warmup 3 --set "sampler=$S" > gpurun_out/prof_s$S.log 2>&1
done
ls -la gpurun_out
