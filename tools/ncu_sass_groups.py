"""Per-opcode totals of a kernel's SASS source page (ncu --page source
--print-source sass): instructions executed, shared-memory wavefronts (and
the ideal count), warp-stall samples.  Usage:
    python tools/ncu_sass_groups.py rep.ncu-rep kernel-regex [min-address] [max-address]"""
import csv
import io
import subprocess
import sys
from collections import defaultdict


def load(path, kern):
    out = subprocess.run(["ncu", "-i", path, "--page", "source", "--csv", "--print-source", "sass", "-k",
                          f"regex:{kern}"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hi = next(i for i, r in enumerate(rows) if "Address" in r and "Source" in r)
    hdr = rows[hi]
    return hdr, [r for r in rows[hi + 1:] if len(r) == len(hdr) and r[0] != "Address"]


def f(x):
    try:
        return float(x)
    except ValueError:
        return 0.0


def main(path, kern, lo=None, hi=None):
    hdr, data = load(path, kern)
    ix = {h: i for i, h in enumerate(hdr)}
    g = defaultdict(lambda: [0.0] * 5)
    for r in data:
        a = int(r[ix["Address"]], 16) if r[ix["Address"]].startswith("0x") else int(r[ix["Address"]])
        if (lo is not None and a < lo) or (hi is not None and a >= hi):
            continue
        op = r[ix["Source"]].strip().split(" ")[0]
        if op.startswith("@"):
            op = r[ix["Source"]].strip().split(" ")[1]
        op = op.split(".")[0]
        v = g[op]
        v[0] += f(r[ix["Instructions Executed"]])
        v[1] += f(r[ix["L1 Wavefronts Shared"]])
        v[2] += f(r[ix["L1 Wavefronts Shared Ideal"]])
        v[3] += f(r[ix["Warp Stall Sampling (All Samples)"]])
        v[4] += f(r[ix["L2 Theoretical Sectors Global"]])
    tot = [sum(v[i] for v in g.values()) or 1 for i in range(5)]
    print(f"{'op':10s} {'inst%':>7s} {'shWF%':>7s} {'shWF/ideal':>10s} {'stall%':>7s} {'L2sec%':>7s}")
    for op, v in sorted(g.items(), key=lambda kv: -kv[1][3])[:30]:
        print(f"{op:10s} {100*v[0]/tot[0]:7.2f} {100*v[1]/tot[1]:7.2f} {v[1]/max(v[2],1):10.2f} "
              f"{100*v[3]/tot[3]:7.2f} {100*v[4]/tot[4]:7.2f}")
    print(f"total inst {tot[0]:.4g}, shared wavefronts {tot[1]:.4g} (ideal {tot[2]:.4g}), L2 sectors {tot[4]:.4g}")


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2], *(int(x, 0) for x in sys.argv[3:5]))
