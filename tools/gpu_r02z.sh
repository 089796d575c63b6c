# per-kernel device time of the PubMed load path (a0)
OUT=gpurun_out; mkdir -p $OUT
LDA_TIMING=1 python tools/load_only.py --config pubmed > $OUT/r02z_load.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -k 'regex:^(layout_keys_kernel|rs_hist_kernel|rs_scatter_kernel|scan_|invert_kernel|tok_row_kernel|init_tile_kernel|recount_kernel|theta_kernel|gather_z_kernel|zero_rows_kernel)' --csv --log-file $OUT/r02z_load_launches.csv python tools/load_only.py --config pubmed --reps 1 > $OUT/r02z_ncu.log 2>&1
python - <<'P'
import csv, collections
rows = list(csv.DictReader(l for l in open("gpurun_out/r02z_load_launches.csv") if l.startswith('"')))
agg = collections.defaultdict(lambda: [0, 0.0])
for r in rows:
    if r.get("Metric Name") == "gpu__time_duration.sum":
        v = float(r["Metric Value"].replace(",", ""))
        unit = r.get("Metric Unit", "")
        ms = v / 1e6 if unit == "nsecond" else v / 1e3 if unit == "usecond" else v
        k = r["Kernel Name"].split("(")[0]
        agg[k][0] += 1; agg[k][1] += ms
for k, (n, ms) in sorted(agg.items(), key=lambda x: -x[1][1]):
    print(f"{k:40s} {n:4d} {ms:9.3f} ms")
P
cat $OUT/r02z_load.log | grep -v "^\[lda\] *layout:"
