"""Parity at BASELINE.json's full size, in the launch configuration bench.py
times (-m gpu): the PubMed-shaped corpus (T = 737,869,083, D = 8.2 M,
V = 141,043, K = 1024), generated exactly as bench.py generates it.

The oracle cannot run whole sweeps at this size, so:
  * init (t = 0) is integer: GPU n_wk, n_k must equal the oracle's init counts
    bit for bit over the WHOLE corpus (one Philox draw per token per word
    range), and sampled tokens' z must equal the oracle's;
  * sweep 1 is checked on sampled tokens: the oracle draws each one from the
    exact init counts (its word's n_wk row, n_k, its document's n_dk row);
  * later sweeps are checked by the count invariants, which hold at any size.
"""
import numpy as np
import pytest
import torch

import lda_testutil as U
from oracle import oracle as O
import paper_conf_hpdc_xie0lt19_b200 as L
from paper_conf_hpdc_xie0lt19_b200 import config as C
from paper_conf_hpdc_xie0lt19_b200 import synth

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def pubmed():
    cfg = synth.CONFIGS["pubmed"]
    dp, w, _ = synth.generate_config(cfg, torch.device("cuda", 0))
    doc_ptr, words = synth.to_numpy(dp, w)
    del dp, w
    torch.cuda.empty_cache()
    m = L.LDA(cfg.D, cfg.V, cfg.K, cfg.alpha, cfg.beta, device=0, **C.BENCH_OPTIONS)
    m.load(doc_ptr, words, cfg.seed)
    yield cfg, doc_ptr, words, m
    m.close()


def test_fullsize_init_and_sweep1_sampled(pubmed):
    cfg, doc_ptr, words, m = pubmed
    K, V, T = cfg.K, cfg.V, cfg.T
    assert int(doc_ptr[-1]) == T and len(doc_ptr) == cfg.D + 1

    # --- init counts, whole corpus, bit-exact
    wc = np.bincount(words, minlength=V).astype(np.int64)
    wstart = np.concatenate([[0], np.cumsum(wc)])
    nwk_o = np.zeros((V, K), np.int32)
    for w in range(V):
        if wc[w]:
            O.init_range_hist(cfg.seed, int(wstart[w]), int(wc[w]), K, nwk_o[w])
    nk_o = nwk_o.sum(0, dtype=np.int64).astype(np.int32)
    nwk_g = m.nwk()
    assert np.array_equal(nwk_g, nwk_o)
    assert np.array_equal(m.nk(), nk_o)
    z0_g = m.z()

    # --- sampled documents: canonical indices, z0 and n_dk rows
    rng = np.random.default_rng(2024)
    docs = np.sort(rng.choice(cfg.D, size=600, replace=False))
    tok = np.concatenate([np.arange(doc_ptr[d], doc_ptr[d + 1]) for d in docs])
    canon = O.canonical_index_of(doc_ptr, words, V, tok)
    z0_o = np.array([O.init_topic(cfg.seed, int(c), K) for c in canon], np.uint16)
    assert np.array_equal(z0_g[tok], z0_o)
    ptr, top, cnt = m.theta_csr()
    off = 0
    ndk_rows = {}
    for d in docs:
        n = int(doc_ptr[d + 1] - doc_ptr[d])
        row = np.zeros(K, np.int32)
        np.add.at(row, z0_o[off:off + n].astype(np.int64), 1)
        g = np.zeros(K, np.int32)
        g[top[ptr[d]:ptr[d + 1]].astype(np.int64)] = cnt[ptr[d]:ptr[d + 1]]
        assert np.array_equal(g, row), d
        ndk_rows[d] = row
        off += n

    # --- sweep 1 on the sampled tokens
    m.iterate(1)
    z1_g = m.z()
    doc_of = np.repeat(docs, np.diff(doc_ptr)[docs])
    bad = unexcused = 0
    for i, c, d in zip(tok, canon, doc_of):
        x0 = O.token_x0(cfg.seed, int(c), 1)
        z, margin = O.draw(K, V, cfg.alpha, cfg.beta, nwk_o[words[i]], nk_o, ndk_rows[d], x0)
        if z != z1_g[i]:
            bad += 1
            unexcused += margin >= U.MARGIN_EXCUSE
    assert unexcused == 0
    assert bad <= max(1, U.MAX_EXCUSED_FRAC * len(tok))

    # --- more sweeps: invariants at full size
    m.iterate(2)
    U.check_invariants_gpu(m, doc_ptr, words)
    ll = m.loglik()
    assert -15.0 < ll < 0.0
