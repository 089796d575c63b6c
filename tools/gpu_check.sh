# quick full check: GPU suite + smoke + a short bench line
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 600 python bench.py --steps 10 --no-cpu-baseline 2>/dev/null | python -c "import sys,json; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(round(d['value']/1e9,3), 'G tok/s', round(d['roofline']['frac'],3), d['phases_ms_per_step'], d['e2e']['value']/1e9)"
