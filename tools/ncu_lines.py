"""Per-CUDA-line totals of a kernel (ncu --page source --print-source cuda,sass;
needs -lineinfo): instructions executed, warp-stall samples, shared-memory
wavefronts, grouped by source line and by the enclosing function of
kernels.cu.  Usage: python tools/ncu_lines.py rep.ncu-rep kernel-regex [n]"""
import csv
import io
import re
import subprocess
import sys
from collections import defaultdict


def f(x):
    try:
        return float(x)
    except ValueError:
        return 0.0


def main(path, kern, n=40):
    out = subprocess.run(["ncu", "-i", path, "--page", "source", "--csv", "--print-source", "cuda,sass", "-k",
                          f"regex:{kern}"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hi = next(i for i, r in enumerate(rows) if r and r[0] == "Line No")
    hdr = rows[hi]
    ix = {}
    for i, h in enumerate(hdr):
        ix.setdefault(h, i)
    sass_src = [i for i, h in enumerate(hdr) if h == "Source"][1]
    per = defaultdict(lambda: [0.0, 0.0, 0.0, ""])
    line = None
    for r in rows[hi + 1:]:
        if len(r) < len(hdr):
            continue
        if r[0].strip().isdigit():
            line = int(r[0])
            per[line][3] = r[1].strip()[:70]
        if not r[ix["Address"]].strip() or line is None:
            continue
        v = per[line]
        v[0] += f(r[ix["Instructions Executed"]])
        v[1] += f(r[ix["Warp Stall Sampling (All Samples)"]])
        v[2] += f(r[ix["L1 Wavefronts Shared"]])
    src = open(sys.argv[4] if len(sys.argv) > 4 else "paper_conf_hpdc_xie0lt19_b200/csrc/kernels.cu").read().split("\n")
    # enclosing function of each line: last line matching a function header
    fn_at, cur = {}, "?"
    pat = re.compile(r"^(?:template.*)?(?:__device__|__global__).*?\b(\w+)\s*\(")
    for i, s in enumerate(src, 1):
        m = pat.match(s)
        if m:
            cur = m.group(1)
        fn_at[i] = cur
    tot = [sum(v[k] for v in per.values()) or 1 for k in range(3)]
    byfn = defaultdict(lambda: [0.0, 0.0, 0.0])
    for ln, v in per.items():
        for k in range(3):
            byfn[fn_at.get(ln, "?")][k] += v[k]
    print("by function:            inst%  stall%  shWF%")
    for fn, v in sorted(byfn.items(), key=lambda kv: -kv[1][1]):
        print(f"  {fn:22s} {100*v[0]/tot[0]:6.2f} {100*v[1]/tot[1]:6.2f} {100*v[2]/tot[2]:6.2f}")
    print(f"top lines by stall samples (inst% stall% shWF%):")
    for ln, v in sorted(per.items(), key=lambda kv: -kv[1][1])[:n]:
        print(f"  {ln:5d} {100*v[0]/tot[0]:6.2f} {100*v[1]/tot[1]:6.2f} {100*v[2]/tot[2]:6.2f}  {v[3]}")


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2], int(sys.argv[3]) if len(sys.argv) > 3 else 40)
