cat /sys/kernel/mm/transparent_hugepage/enabled /sys/kernel/mm/transparent_hugepage/defrag
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "nytimes_shaped or edge or tile_sampler" 2>&1 | tail -2
LDA_TIMING=1 timeout 300 python tools/exp_options.py --sweeps 5 --set "sampler=2" 2>&1 | grep -v "^#"
