timeout 300 python tools/exp_options.py --sweeps 5 --set "sampler=2" 2>&1 | grep -v "^#" | cut -c 1-150
LDA_NO_DOC_SORT=1 timeout 300 python tools/exp_options.py --sweeps 5 --set "sampler=2" 2>&1 | grep -v "^#" | cut -c 1-150
LDA_NO_DOC_SORT=1 timeout 300 python tools/exp_options.py --config nytimes --sweeps 5 --set "sampler=2" 2>&1 | grep -v "^#" | cut -c 1-150
timeout 300 python tools/exp_options.py --config nytimes --sweeps 5 --set "sampler=2" 2>&1 | grep -v "^#" | cut -c 1-150
