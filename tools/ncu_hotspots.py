"""Top SASS lines by warp-stall samples from an ncu report (needs -lineinfo).
Usage: python tools/ncu_hotspots.py rep.ncu-rep [kernel-substring] [n]"""
import csv
import io
import subprocess
import sys


def main(path, kern=None, n=25):
    args = ["ncu", "-i", path, "--page", "source", "--csv", "--print-source", "sass"]
    if kern:
        args += ["-k", f"regex:{kern}"]
    out = subprocess.run(args, capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr_i = next(i for i, r in enumerate(rows) if "Address" in r and "Source" in r)
    hdr = rows[hdr_i]
    ix = {h: i for i, h in enumerate(hdr)}
    data = [r for r in rows[hdr_i + 1:] if len(r) == len(hdr) and r[0] != "Address"]
    key = "Warp Stall Sampling (All Samples)"
    tot = sum(float(r[ix[key]] or 0) for r in data) or 1.0
    stall_cols = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
    for r in sorted(data, key=lambda r: -float(r[ix[key]] or 0))[:n]:
        st = sorted(((float(r[ix[c]] or 0), c[6:]) for c in stall_cols), reverse=True)[:2]
        print(f"{float(r[ix[key]] or 0) / tot * 100:5.1f}%  {r[ix['Address']]:>6s} {r[ix['Source']][:64]:64s} "
              + " ".join(f"{c}={v:.0f}" for v, c in st))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else None, int(sys.argv[3]) if len(sys.argv) > 3 else 25)
