OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -m gpu -q -x -p no:cacheprovider -k "radix or appendix or tiny_config_lockstep or edge_cases or midsize or fullsize" > $OUT/r02ae_pytest.log 2>&1; echo "pytest exit $?" >> $OUT/r02ae_pytest.log
tail -3 $OUT/r02ae_pytest.log
LDA_TIMING=1 python tools/load_only.py --config pubmed --reps 3 --pinned > $OUT/r02ae_load_pinned.log 2>&1
grep -E "sorter|copiers|load [0-9]" $OUT/r02ae_load_pinned.log
ncu --metrics gpu__time_duration.sum --clock-control none -k 'regex:(layout_keys_kernel|rs_hist_kernel|rs_scatter_kernel|scan_|invert_kernel)' --csv --log-file $OUT/r02ae_load_launches.csv python tools/load_only.py --config pubmed --reps 1 --pinned > $OUT/r02ae_ncu.log 2>&1
python - <<'P'
import csv, collections
rows = list(csv.DictReader(l for l in open("gpurun_out/r02ae_load_launches.csv") if l.startswith('"')))
agg = collections.defaultdict(lambda: [0, 0.0])
for r in rows:
    if r.get("Metric Name") == "gpu__time_duration.sum":
        v = float(r["Metric Value"].replace(",", "")); u = r.get("Metric Unit", "")
        ms = v / 1e6 if u in ("ns", "nsecond") else v / 1e3 if u in ("us", "usecond") else v
        k = r["Kernel Name"].split("(")[0]
        agg[k][0] += 1; agg[k][1] += ms
for k, (n, ms) in sorted(agg.items(), key=lambda x: -x[1][1]):
    print(f"{k:60s} {n:4d} {ms:9.3f} ms")
P
