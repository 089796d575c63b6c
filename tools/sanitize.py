"""Small runs of every sampler and path for compute-sanitizer (memcheck /
racecheck / synccheck):
    compute-sanitizer --tool racecheck python tools/sanitize.py"""
import os
import sys
import threading

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_hpdc_xie0lt19_b200 as L  # noqa: E402
from paper_conf_hpdc_xie0lt19_b200 import synth  # noqa: E402

doc_ptr, words = synth.to_numpy(*synth.generate(300, 400, 20_000, 0.7, 16, 7, "cpu"))[:2]
for K, opts in [(64, dict(sampler=2, tile_tokens=5000)), (64, dict(sampler=3, tile_tokens=5000)),
                (64, dict(sampler=2, fused_recount=1, tile_tokens=5000)), (37, dict(sampler=2)),
                (5000, dict(sampler=3, tile_tokens=3000)),
                (5000, dict(sampler=3, tile_tokens=3000, sparse_words=-1)),   # f2 sparse word rows
                (5000, dict(sampler=3, sparse_words=1 << 30)), (64, dict(sampler=0)),
                (64, dict(exclude_self=1)), (20000, {}), (64, dict(stream_chunks=3, tile_tokens=5000)),
                (64, dict(sampler=2, certify_slack=1 << 20))]:
    m = L.LDA(300, 400, K, 50.0 / K, 0.01, loglik_every=2, **opts).load(doc_ptr, words, 3)
    m.iterate(2)
    z = m.z()
    m.set_z(z)
    print(K, opts, "LL", round(m.loglik(), 5), flush=True)
    m.close()

# two ranks of an in-process peer group (the P2P exchange kernels)
bounds = L.lda_partition_docs(doc_ptr, 2)
grp = L.PeerGroup(2)


def rank(r):
    d0, d1 = int(bounds[r]), int(bounds[r + 1])
    t0, t1 = int(doc_ptr[d0]), int(doc_ptr[d1])
    m = L.LDA(300, 400, 64, 50.0 / 64, 0.01, comm_pipeline=3)
    m.init_peer(grp, r)
    m.load(doc_ptr[d0:d1 + 1] - t0, words[t0:t1], 3, d0, d1)
    m.iterate(2)
    print("peer rank", r, "LL", round(m.loglik(), 5), flush=True)
    m.close()


th = [threading.Thread(target=rank, args=(r,)) for r in range(2)]
for t in th:
    t.start()
for t in th:
    t.join()
grp.close()
