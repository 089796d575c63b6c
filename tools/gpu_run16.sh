timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
LDA_TIMING=1 timeout 300 python tools/exp_options.py --sweeps 5 --set "sampler=2" 2>&1 | grep -v "^#"
timeout 600 python bench.py --no-cpu-baseline 2>&1 | python -c "import sys,json; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d['value'], d['e2e'], d['roofline']['frac'])"
