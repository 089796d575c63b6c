"""Parity at BASELINE.json's full size, in the launch configuration bench.py
times (-m gpu): the PubMed-shaped corpus (T = 737,869,083, D = 8.2 M,
V = 141,043, K = 1024), generated exactly as bench.py generates it, run with
the library's defaults (bench.py sets no options).

The oracle cannot run whole sweeps at this size, so:
  * init (t = 0) is integer: GPU n_wk, n_k must equal the oracle's init counts
    bit for bit over the WHOLE corpus, and sampled tokens' z must equal the
    oracle's;
  * sweep 1 is checked on sampled tokens drawn by the oracle from the exact
    init counts;
  * in the benchmarked regime (the bench times sweeps 24-43): after sweep 25
    n_wk, n_k are recounted from the GPU's z by brute force on the host (whole
    corpus, bit-exact) and θ is checked against it; then >= 10^6 tokens of
    sampled documents are drawn by the oracle for sweep 26 from that exact
    state (teacher forcing) and compared with the GPU's draws;
  * the certified fp32 tile sampler (the default) is run against the fp64
    lane-per-token sampler over the WHOLE corpus for 3 sweeps from the same
    state: they may differ only where the oracle's own margin is < 1e-6
    (north_star), in at most 1e-6 of the tokens -- the scale at which a wrong
    certification bound would show.
"""
import numpy as np
import pytest
import torch

import lda_testutil as U
from oracle import oracle as O
import paper_conf_hpdc_xie0lt19_b200 as L
from paper_conf_hpdc_xie0lt19_b200 import synth

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def pubmed():
    cfg = synth.CONFIGS["pubmed"]
    dp, w, _ = synth.generate_config(cfg, torch.device("cuda", 0))
    doc_ptr, words = synth.to_numpy(dp, w)
    del dp, w
    torch.cuda.empty_cache()
    m = L.LDA(cfg.D, cfg.V, cfg.K, cfg.alpha, cfg.beta, device=0)
    m.load(doc_ptr, words, cfg.seed)
    yield cfg, doc_ptr, words, m
    m.close()


def _host_counts(words, z, V, K, chunk=50_000_000):
    """n_wk, n_k recounted from z by brute force (numpy bincount)."""
    nwk = np.zeros(V * K, np.int64)
    for i in range(0, len(words), chunk):
        key = words[i:i + chunk].astype(np.int64) * K + z[i:i + chunk].astype(np.int64)
        nwk += np.bincount(key, minlength=V * K)
    nwk = nwk.reshape(V, K)
    return nwk, nwk.sum(0)


def _sample_docs(doc_ptr, n_tokens, seed):
    rng = np.random.default_rng(seed)
    D = len(doc_ptr) - 1
    docs = np.unique(rng.choice(D, size=int(1.3 * n_tokens / max(1.0, doc_ptr[-1] / D)), replace=False))
    L_d = np.diff(doc_ptr)[docs]
    keep = np.searchsorted(np.cumsum(L_d), n_tokens) + 1
    return docs[:keep]


def _sub_corpus(doc_ptr, words, docs, V):
    """Sampled documents as a sub-corpus: offsets, words, input positions and
    the GLOBAL canonical index of every token."""
    L_d = np.diff(doc_ptr)[docs]
    sub_ptr = np.concatenate([[0], np.cumsum(L_d)]).astype(np.int64)
    tok = np.concatenate([np.arange(doc_ptr[d], doc_ptr[d + 1]) for d in docs]).astype(np.int64)
    canon = O.canonical_index_of(doc_ptr, words, V, tok)
    return sub_ptr, np.ascontiguousarray(words[tok]), tok, canon


def _dense_rows(sub_ptr, z_sub, K):
    nd = len(sub_ptr) - 1
    rows = np.zeros((nd, K), np.int32)
    doc_of = np.repeat(np.arange(nd), np.diff(sub_ptr))
    np.add.at(rows, (doc_of, z_sub.astype(np.int64)), 1)
    return rows


def test_fullsize_init_and_sweep1_sampled(pubmed):
    cfg, doc_ptr, words, m = pubmed
    K, V, T = cfg.K, cfg.V, cfg.T
    assert int(doc_ptr[-1]) == T and len(doc_ptr) == cfg.D + 1
    st = m.stats()
    assert st["sampler"] == 2 and st["n_tiles"] > 1, st      # the bench's path: tile sampler, auto tiles

    # --- init counts, whole corpus, bit-exact
    wc = np.bincount(words, minlength=V).astype(np.int64)
    wstart = np.concatenate([[0], np.cumsum(wc)])
    nwk_o = np.zeros((V, K), np.int32)
    for w in range(V):
        if wc[w]:
            O.init_range_hist(cfg.seed, int(wstart[w]), int(wc[w]), K, nwk_o[w])
    nk_o = nwk_o.sum(0, dtype=np.int64).astype(np.int32)
    assert np.array_equal(m.nwk(), nwk_o)
    assert np.array_equal(m.nk(), nk_o)
    z0_g = m.z()

    # --- sampled documents: canonical indices, z0 and n_dk rows
    docs = _sample_docs(doc_ptr, 60_000, 2024)
    sub_ptr, sub_words, tok, canon = _sub_corpus(doc_ptr, words, docs, V)
    z0_o = np.array([O.init_topic(cfg.seed, int(c), K) for c in canon], np.uint16)
    assert np.array_equal(z0_g[tok], z0_o)
    ptr, top, cnt = m.theta_csr()
    rows0 = _dense_rows(sub_ptr, z0_o, K)
    for j, d in enumerate(docs):
        g = np.zeros(K, np.int32)
        g[top[ptr[d]:ptr[d + 1]].astype(np.int64)] = cnt[ptr[d]:ptr[d + 1]]
        assert np.array_equal(g, rows0[j]), d

    # --- sweep 1 on the sampled tokens, drawn by the oracle from the init state
    m.iterate(1)
    z1_g = m.z()
    z1_o, margin = O.draw_docs(0, len(docs), sub_ptr, sub_words, canon, V, K, cfg.alpha, cfg.beta, cfg.seed, 1,
                               z0_o, nwk_o, nk_o, rows0, margins=True)
    bad = np.nonzero(z1_g[tok] != z1_o)[0]
    assert (margin[bad] < U.MARGIN_EXCUSE).all()
    assert len(bad) <= max(1, U.MAX_EXCUSED_FRAC * len(tok))


def test_fullsize_benchmarked_regime(pubmed):
    """Sweeps 25-26 (inside the bench's timed window): whole-corpus brute-force
    recount, θ, and >= 10^6 teacher-forced oracle draws."""
    cfg, doc_ptr, words, m = pubmed
    K, V, T = cfg.K, cfg.V, cfg.T
    m.iterate(25 - m.stats()["sweeps_done"])
    assert m.stats()["sweeps_done"] == 25
    z25 = m.z()
    # (i) n_wk, n_k from z by brute force: bit-exact
    nwk_h, nk_h = _host_counts(words, z25, V, K)
    nwk_g = m.nwk()
    assert np.array_equal(nwk_g, nwk_h)
    assert np.array_equal(m.nk(), nk_h)
    # θ: invariants over every document, Σ_d n_dk = n_k per topic, exact rows
    # of sampled documents
    U.check_invariants_gpu(m, doc_ptr, words)
    ptr, top, cnt = m.theta_csr()
    assert np.array_equal(np.bincount(top, weights=cnt, minlength=K).astype(np.int64), nk_h)
    docs = _sample_docs(doc_ptr, 1_000_000, 77)
    sub_ptr, sub_words, tok, canon = _sub_corpus(doc_ptr, words, docs, V)
    assert len(tok) >= 1_000_000
    rows25 = _dense_rows(sub_ptr, z25[tok], K)
    for j in range(0, len(docs), 97):
        d = docs[j]
        g = np.zeros(K, np.int32)
        g[top[ptr[d]:ptr[d + 1]].astype(np.int64)] = cnt[ptr[d]:ptr[d + 1]]
        assert np.array_equal(g, rows25[j]), d
    del ptr, top, cnt
    # (ii) sweep 26: the oracle's draws of the sampled tokens from the exact
    # sweep-25 state vs the GPU's
    m.iterate(1)
    z26_g = m.z()
    z26_o, margin = O.draw_docs(0, len(docs), sub_ptr, sub_words, canon, V, K, cfg.alpha, cfg.beta, cfg.seed,
                                26, z25[tok], nwk_g.astype(np.int32), nk_h.astype(np.int32), rows25,
                                margins=True)
    bad = np.nonzero(z26_g[tok] != z26_o)[0]
    assert (margin[bad] < U.MARGIN_EXCUSE).all(), margin[bad]
    assert len(bad) <= max(1, U.MAX_EXCUSED_FRAC * len(tok))


def test_fullsize_certified_fp32_vs_fp64_sampler(pubmed):
    """(iii) The default sampler's fp32 draws are certified against rigorous
    bounds (X24); the lane-per-token sampler draws in fp64.  Over
    the whole 738 M-token corpus for 3 sweeps from the same state they may
    differ only within fp64 rounding of a CDF boundary: every mismatch is
    excused by the oracle's margin (< 1e-6) and mismatches are <= 1e-6 of T."""
    cfg, doc_ptr, words, m = pubmed
    K, V, T = cfg.K, cfg.V, cfg.T
    f = L.LDA(cfg.D, cfg.V, cfg.K, cfg.alpha, cfg.beta, device=0, sampler=0)
    f.load(doc_ptr, words, cfg.seed)
    try:
        t = m.stats()["sweeps_done"]
        f.iterate(t)                    # the same sweep counter (Philox key word) ...
        z = m.z()
        f.set_z(z)                      # ... and the same state
        total_bad = 0
        for _ in range(3):
            nwk_prev, nk_prev = m.nwk(), m.nk()
            m.iterate(1)
            f.iterate(1)
            t += 1
            za, zb = m.z(), f.z()
            bad = np.nonzero(za != zb)[0]
            total_bad += len(bad)
            assert len(bad) <= 1e-6 * T + 2
            if len(bad):
                # the oracle on the documents of the mismatched tokens
                docs = np.unique(np.searchsorted(doc_ptr, bad, side="right") - 1)
                sub_ptr, sub_words, tok, canon = _sub_corpus(doc_ptr, words, docs, V)
                rows = _dense_rows(sub_ptr, z[tok], K)
                _, margin = O.draw_docs(0, len(docs), sub_ptr, sub_words, canon, V, K, cfg.alpha, cfg.beta,
                                        cfg.seed, t, z[tok], nwk_prev, nk_prev, rows, margins=True)
                pos = {int(i): j for j, i in enumerate(tok)}
                mb = np.array([margin[pos[int(i)]] for i in bad])
                assert (mb < U.MARGIN_EXCUSE).all(), mb
                f.set_z(za)             # keep the chains in lock step
            z = za
        print(f"fp32-certified vs fp64 sampler: {total_bad} differing draws in 3 x {T} tokens")
    finally:
        f.close()
    U.check_invariants_gpu(m, doc_ptr, words)
    ll = m.loglik()
    assert -15.0 < ll < 0.0
