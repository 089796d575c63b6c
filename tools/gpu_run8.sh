mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "exact_redraw or tile_sampler" > gpurun_out/gpu_tests10.log 2>&1; tail -2 gpurun_out/gpu_tests10.log
for c in nytimes_k128 nytimes nytimes_k8192; do
timeout 400 python tools/exp_options.py --config $c --sweeps 5 --set "sampler=2,tile_tokens=16000000" --set "sampler=2,tile_tokens=8000000" --set "sampler=0" 2>&1 | grep -v "^#" | sed "s/^/$c /"
done
