import json,sys
for line in sys.stdin:
    line=line.strip()
    if not line.startswith("{"): continue
    d=json.loads(line)
    print(round(d["value"]/1e9,3), {k:round(v,2) for k,v in d["phases_ms_per_step"].items()}, "frac", round(d["roofline"]["frac"],3), "nnz", round(d["nnz_per_token"],1), d["config"]["options"])
