"""Markdown summary of an ncu report of the sampling kernel (for profiles/):
the raw metrics of tools/ncu_summary.py, the per-function and per-line
instruction / stall / shared-wavefront split of tools/ncu_lines.py and the
SASS opcode groups of tools/ncu_sass_groups.py.
Usage: python tools/profile_md.py rep.ncu-rep kernel-regex title > profiles/X.md"""
import contextlib
import io
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import ncu_lines  # noqa: E402
import ncu_sass_groups  # noqa: E402
import ncu_summary  # noqa: E402


def grab(f, *a):
    buf = io.StringIO()
    with contextlib.redirect_stdout(buf):
        f(*a)
    return buf.getvalue()


def main(rep, kern, title):
    print(f"# {title}\n\nReport: `{os.path.basename(rep)}` (ncu --set full --import-source on, "
          f"--clock-control none; one launch)\n")
    print("## Metrics\n\n```\n" + grab(ncu_summary.main, rep) + "```\n")
    print("## Instructions / stall samples / shared wavefronts by source function and line\n\n```\n"
          + grab(ncu_lines.main, rep, kern, 30) + "```\n")
    print("## SASS opcode groups\n\n```\n" + grab(ncu_sass_groups.main, rep, kern) + "```")


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2], sys.argv[3])
