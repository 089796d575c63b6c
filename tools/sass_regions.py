"""Instruction / stall / shared-wavefront share per 40-SASS-instruction region of one kernel.
Usage: python tools/sass_regions.py rep kernel-regex [region]"""
import csv, io, subprocess, sys
rep, kern = sys.argv[1], sys.argv[2]
R = int(sys.argv[3]) if len(sys.argv) > 3 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass", "-k", "regex:" + kern],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hi = next(i for i, r in enumerate(rows) if 'Address' in r)
h = rows[hi]; ix = {k: i for i, k in enumerate(h)}
data = [r for r in rows[hi + 1:] if len(r) == len(h) and r[0] != 'Address']
def f(r, k):
    try:
        return float(r[ix[k]] or 0)
    except ValueError:
        return 0.0
ti = sum(f(r, 'Instructions Executed') for r in data)
ts = sum(f(r, 'Warp Stall Sampling (All Samples)') for r in data)
tw = sum(f(r, 'L1 Wavefronts Shared') for r in data) or 1
stcols = [c for c in h if c.startswith('stall_') and 'Not Issued' not in c]
for s in range(0, len(data), R):
    ch = data[s:s + R]
    pi = sum(f(r, 'Instructions Executed') for r in ch) / ti * 100
    ps = sum(f(r, 'Warp Stall Sampling (All Samples)') for r in ch) / ts * 100
    pw = sum(f(r, 'L1 Wavefronts Shared') for r in ch) / tw * 100
    if pi > 0.5 or ps > 0.5 or pw > 0.5:
        top = sorted(((sum(f(r, c) for r in ch), c[6:]) for c in stcols), reverse=True)[:3]
        print(f"{s:5d} inst {pi:5.1f}% stall {ps:5.1f}% shwf {pw:5.1f}% {ch[0][ix['Source']].strip()[:30]:30s} | "
              + " ".join(f"{c}={v / ts * 100:.1f}" for v, c in top))
