"""Small runs of every sampler for compute-sanitizer (memcheck / racecheck):
    compute-sanitizer --tool racecheck python tools/sanitize.py"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_hpdc_xie0lt19_b200 as L  # noqa: E402
from paper_conf_hpdc_xie0lt19_b200 import synth  # noqa: E402

doc_ptr, words = synth.to_numpy(*synth.generate(300, 400, 20_000, 0.7, 16, 7, "cpu"))[:2]
for K, opts in [(64, dict(sampler=2, tile_tokens=5000)), (64, dict(sampler=3, tile_tokens=5000)),
                (64, dict(sampler=2, fused_recount=1, tile_tokens=5000)), (37, dict(sampler=2)),
                (5000, dict(sampler=3, tile_tokens=3000)), (64, dict(sampler=0))]:
    m = L.LDA(300, 400, K, 50.0 / K, 0.01, **opts).load(doc_ptr, words, 3)
    m.iterate(2)
    z = m.z()
    m.set_z(z)
    print(K, opts, "LL", round(m.loglik(), 5), flush=True)
    m.close()
