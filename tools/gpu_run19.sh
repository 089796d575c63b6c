timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -k "k_variants or edge or tile_sampler or k8192 or exact_redraw" 2>&1 | tail -3
timeout 300 python tools/exp_options.py --sweeps 5 --set "sampler=2" --set "sampler=3" 2>&1 | grep -v "^#"
for c in nytimes_k128 nytimes nytimes_k8192; do
timeout 400 python tools/exp_options.py --config $c --sweeps 5 --set "sampler=2" --set "sampler=3" --set "sampler=0" 2>&1 | grep -v "^#" | sed "s/^/$c /"
done
