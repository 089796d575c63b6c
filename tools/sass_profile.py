"""Instruction / stall distribution over the SASS of one kernel (ncu report).
Usage: python tools/sass_profile.py rep kernel-regex [min_pct]"""
import csv, io, subprocess, sys
rep, kern = sys.argv[1], sys.argv[2]
minp = float(sys.argv[3]) if len(sys.argv) > 3 else 0.6
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass", "-k", "regex:" + kern],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hi = next(i for i, r in enumerate(rows) if 'Address' in r)
h = rows[hi]; ix = {k: i for i, k in enumerate(h)}
data = [r for r in rows[hi + 1:] if len(r) == len(h)]
f = lambda r, k: float(r[ix[k]] or 0)
ti = sum(f(r, 'Instructions Executed') for r in data)
ts = sum(f(r, 'Warp Stall Sampling (All Samples)') for r in data)
tw = sum(f(r, 'L1 Wavefronts Shared') for r in data)
print(f"total inst {ti:.3e}  shared wavefronts {tw:.3e}")
for n, r in enumerate(data):
    pi = f(r, 'Instructions Executed') / ti * 100
    ps = f(r, 'Warp Stall Sampling (All Samples)') / ts * 100
    pw = f(r, 'L1 Wavefronts Shared') / tw * 100 if tw else 0
    if pi >= minp or ps >= minp or pw >= minp:
        print(f"{n:5d} inst {pi:5.2f}% stall {ps:5.2f}% shwf {pw:5.2f}% thr {f(r,'Avg. Threads Executed'):4.1f}  {r[ix['Source']].strip()[:70]}")
