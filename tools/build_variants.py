"""Build compile-time variants of liblda.so under variants/ (git-ignored,
shipped to the GPU box by gpurun) for A/B timing with LDA_LIBRARY=...
Usage: python tools/build_variants.py name:DEF=1,DEF2=0 ..."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_hpdc_xie0lt19_b200 import _build  # noqa: E402

if __name__ == "__main__":
    os.makedirs(os.path.join(ROOT, "variants"), exist_ok=True)
    for spec in sys.argv[1:]:
        name, _, defs = spec.partition(":")
        out = os.path.join(ROOT, "variants", f"liblda_{name}.so")
        _build.build(out=out, defines=[d for d in defs.split(",") if d])
        print(out)
