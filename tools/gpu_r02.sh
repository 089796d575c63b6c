# round-2 GPU check: the whole -m gpu suite (durations), smoke, a short bench line
mkdir -p gpurun_out
tag=${1:-r02}
timeout 2400 python -m pytest tests -m gpu -q -rA --durations=15 -p no:cacheprovider > gpurun_out/${tag}_pytest.log 2>&1
echo "pytest exit $?" >> gpurun_out/${tag}_pytest.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${tag}_smoke.log 2>&1
timeout 900 python bench.py --steps 20 --warmup 3 > gpurun_out/${tag}_bench.json 2> gpurun_out/${tag}_bench.err
tail -3 gpurun_out/${tag}_pytest.log
tail -1 gpurun_out/${tag}_smoke.log
