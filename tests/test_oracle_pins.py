"""Pins of the CPU oracle against things other than itself (-m "not gpu").

Each test names what fixes the expected value: a Random123 KAT, the paper's
Fig. 5 worked example, SURVEY.md Appendix A (an independent implementation),
a closed form, or a brute-force recomputation along a different route.
"""
import json
import math
import os

import numpy as np
import pytest
from scipy.special import gammaln

from oracle import oracle as O
GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def _golden(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


def _micro():
    g = _golden("appendix_a_micro.json")
    words = np.array(sum(g["docs"], []), np.int32)
    doc_ptr = np.cumsum([0] + [len(d) for d in g["docs"]]).astype(np.int64)
    return g, doc_ptr, words


# --------------------------------------------------------------------------
# Philox4x32-10
# --------------------------------------------------------------------------

def test_philox_known_answers():
    kat = _golden("philox_kat.json")
    for v in kat["vectors"]:
        ctr = [int(x, 16) for x in v["ctr"]]
        key = [int(x, 16) for x in v["key"]]
        out = O.philox4x32_10(ctr, key)
        assert [f"{x:08x}" for x in out] == v["out"]


def test_token_x0_counter_layout():
    """Counter (c_lo, c_hi, t, 0), key (seed_lo, seed_hi), word x0 (X9):
    checked against the raw block function with a 64-bit c and seed."""
    seed, c, t = 0x1234_5678_9ABC_DEF0, 0x0000_0003_0000_0007, 5
    raw = O.philox4x32_10([c & 0xFFFFFFFF, c >> 32, t, 0],
                          [seed & 0xFFFFFFFF, seed >> 32])
    assert O.token_x0(seed, c, t) == int(raw[0])


def test_appendix_a_x0_streams():
    g, _, _ = _micro()
    for c, hx in enumerate(g["init"]["x0"]):
        assert O.token_x0(g["seed"], c, 0) == int(hx, 16)
    for sw in g["sweeps"]:
        for c, hx in enumerate(sw["x0"]):
            assert O.token_x0(g["seed"], c, sw["t"]) == int(hx, 16)


# --------------------------------------------------------------------------
# Search rule (Fig. 5) and edge cases (X6)
# --------------------------------------------------------------------------

def test_fig5_worked_example():
    f = _golden("fig5_tree_sampling.json")
    prefix = np.cumsum(f["p_x100"]).astype(np.float64)
    assert prefix.tolist() == f["prefix_x100"]
    assert O.search(prefix, f["u_x100"]) == f["k"]
    # The two index-tree levels of Fig. 5 are every 4th / every 2nd prefix.
    assert f["tree_level1_x100"] == [prefix[1], prefix[5]]
    assert f["tree_level2_x100"] == [prefix[0], prefix[2], prefix[4], prefix[6]]


def test_search_edges():
    p = np.array([0.0, 2.0, 2.0, 5.0])
    assert O.search(p, 0.0) == 1          # leading zero-mass bin skipped
    assert O.search(p, 2.0) == 3          # x exactly on a boundary -> next bin
    assert O.search(p, 1.999) == 1
    assert O.search(p, 5.0) == 4          # x >= total -> none (draw falls back to K-1)


def test_draw_fallback_and_zero_mass():
    # K = 2, all mass on the dense part; x0 = 2^32-1 gives U just below 1.
    z, m = O.draw(2, 3, 0.5, 0.1, np.array([0, 0], np.int32), np.array([0, 0], np.int32),
                  np.array([0, 0], np.int32), 0xFFFFFFFF)
    assert z == 1
    z, _ = O.draw(2, 3, 0.5, 0.1, np.array([0, 0], np.int32), np.array([0, 0], np.int32),
                  np.array([0, 0], np.int32), 0)
    assert z == 0


# --------------------------------------------------------------------------
# Appendix A: canonical order, init, sweeps, SEQUENTIAL mode, LL
# --------------------------------------------------------------------------

def test_canonical_order_matches_lexsort():
    g, doc_ptr, words = _micro()
    canon = O.canonical_order(doc_ptr, words, g["V"])
    d = np.repeat(np.arange(g["D"]), np.diff(doc_ptr))
    j = np.arange(len(words)) - doc_ptr[d]
    order = np.lexsort((j, d, words))          # sort by (w, d, j)
    expect = np.empty_like(order)
    expect[order] = np.arange(len(order))
    assert (canon == expect).all()
    wdj = [[int(words[i]), int(d[i]), int(j[i])] for i in order]
    assert wdj == g["canonical_wdj"]


def test_canonical_order_random_corpus():
    rng = np.random.default_rng(7)
    L = rng.integers(0, 30, size=50)
    doc_ptr = np.concatenate([[0], np.cumsum(L)]).astype(np.int64)
    words = rng.integers(0, 17, size=doc_ptr[-1]).astype(np.int32)
    canon = O.canonical_order(doc_ptr, words, 17)
    d = np.repeat(np.arange(50), L)
    j = np.arange(len(words)) - doc_ptr[d]
    order = np.lexsort((j, d, words))
    assert (canon[order] == np.arange(len(words))).all()
    q = rng.choice(len(words), size=40, replace=False)
    assert (O.canonical_index_of(doc_ptr, words, 17, q) == canon[q]).all()


def test_appendix_a_sweeps():
    g, doc_ptr, words = _micro()
    m = O.OracleLDA(g["D"], g["V"], g["K"], g["alpha"], g["beta"]).load(doc_ptr, words, g["seed"])
    inv = np.argsort(m.canon)
    assert m.z[inv].tolist() == g["init"]["z_canonical"]
    assert m.nwk().tolist() == g["init"]["n_wk"]
    assert m.ndk().tolist() == g["init"]["n_dk"]
    assert m.n_k.tolist() == g["init"]["n_k"]
    assert m.loglik() == pytest.approx(g["init"]["ll_per_token"], abs=1e-11)
    for sw in g["sweeps"]:
        margins = m.iterate(1, margins=True)
        assert m.t == sw["t"]
        assert m.z[inv].tolist() == sw["z_canonical"]
        assert m.nwk().tolist() == sw["n_wk"]
        assert m.ndk().tolist() == sw["n_dk"]
        assert m.n_k.tolist() == sw["n_k"]
        assert m.loglik() == pytest.approx(sw["ll_per_token"], abs=1e-11)
        if "min_margin_at_least" in sw:
            assert margins.min() >= sw["min_margin_at_least"]
        if "z_input_order" in sw:
            assert m.z.tolist() == sw["z_input_order"]
        assert m.invariants() == 0


def test_appendix_a_hand_check_token0():
    """Token c=0 (w=0, d=0) at t=1 from the z0 counts, recomputed here
    along the split of Eq. 6-8 written out by hand."""
    g, doc_ptr, words = _micro()
    h = g["hand_check_token0_t1"]
    nwk = np.array(g["init"]["n_wk"]); nk = np.array(g["init"]["n_k"])
    ndk = np.array(g["init"]["n_dk"])
    V, K, a, b = g["V"], g["K"], g["alpha"], g["beta"]
    pstar = (nwk[0] + b) / (nk + V * b)
    assert pstar == pytest.approx(h["pstar"], abs=1e-11)
    sparse = np.cumsum(ndk[0] * pstar)
    dense = sparse[-1] + np.cumsum(a * pstar)
    assert sparse == pytest.approx(h["sparse_prefix"], abs=1e-6)
    assert dense == pytest.approx(h["dense_prefix"], abs=1e-6)
    x0 = O.token_x0(g["seed"], 0, 1)
    U = x0 / 2**32
    assert U == pytest.approx(h["U"], abs=1e-6)
    z, _ = O.draw(K, V, a, b, nwk[0].astype(np.int32), nk.astype(np.int32),
                  ndk[0].astype(np.int32), x0)
    assert z == h["z"]


def test_appendix_a_sequential():
    g, doc_ptr, words = _micro()
    m = O.OracleLDA(g["D"], g["V"], g["K"], g["alpha"], g["beta"]).load(doc_ptr, words, g["seed"])
    inv = np.argsort(m.canon)
    m.iterate(1, mode="sequential")
    assert m.z[inv].tolist() == g["sequential_t1"]["z_canonical"]
    assert m.loglik() == pytest.approx(g["sequential_t1"]["ll_per_token"], abs=1e-11)
    assert m.invariants() == 0


# --------------------------------------------------------------------------
# Counts and invariants
# --------------------------------------------------------------------------

def test_counts_brute_force_and_invariants(tiny_corpus, tiny_cfg):
    doc_ptr, words, _ = tiny_corpus
    c = tiny_cfg
    m = O.OracleLDA(c.D, c.V, c.K, c.alpha, c.beta).load(doc_ptr, words, c.seed)
    for _ in range(3):
        m.iterate(1)
        d = np.repeat(np.arange(c.D), np.diff(doc_ptr))
        nwk = np.zeros((c.V, c.K), np.int64); np.add.at(nwk, (words, m.z), 1)
        ndk = np.zeros((c.D, c.K), np.int64); np.add.at(ndk, (d, m.z), 1)
        assert (m.nwk() == nwk).all()
        assert (m.ndk() == ndk).all()
        assert (m.n_k == nwk.sum(0)).all()
        assert (ndk.sum(1) == np.diff(doc_ptr)).all()      # Eq. 5
        assert m.invariants() == 0
    # the invariant checker itself rejects a broken state
    m.n_wk[0] += 1
    assert m.invariants() != 0


def test_init_is_uniform_over_topics(tiny_corpus, tiny_cfg):
    from scipy.stats import chisquare
    doc_ptr, words, _ = tiny_corpus
    c = tiny_cfg
    m = O.OracleLDA(c.D, c.V, c.K, c.alpha, c.beta).load(doc_ptr, words, c.seed)
    counts = np.bincount(m.z, minlength=c.K)
    assert chisquare(counts).pvalue > 1e-3
    # init_range_hist over a word's canonical range == counts of that word
    start = np.concatenate([[0], np.cumsum(np.bincount(words, minlength=c.V))])
    for w in (0, 7, 499):
        h = O.init_range_hist(c.seed, int(start[w]), int(start[w + 1] - start[w]), c.K)
        assert (h == m.nwk()[w]).all()


# --------------------------------------------------------------------------
# Log-likelihood (X11)
# --------------------------------------------------------------------------

def _polya_sequence_logprob(doc_ptr, words, z, V, K, a, b):
    """log p(w, z) by the Polya-urn chain rule: tokens one at a time, each
    with predictive probability (n_dk^< + a)/(i_d + K a) * (n_wk^< + b)/(n_k^< + V b).
    A different route from the Gamma-function closed form."""
    ndk = {}; nwk = {}; nk = [0] * K
    lp = 0.0
    for d in range(len(doc_ptr) - 1):
        for pos, i in enumerate(range(doc_ptr[d], doc_ptr[d + 1])):
            k, w = int(z[i]), int(words[i])
            lp += math.log((ndk.get((d, k), 0) + a) / (pos + K * a))
            lp += math.log((nwk.get((w, k), 0) + b) / (nk[k] + V * b))
            ndk[(d, k)] = ndk.get((d, k), 0) + 1
            nwk[(w, k)] = nwk.get((w, k), 0) + 1
            nk[k] += 1
    return lp


def test_loglik_polya_chain_rule():
    rng = np.random.default_rng(3)
    for K in (1, 2, 5):
        L = rng.integers(0, 9, size=6)
        doc_ptr = np.concatenate([[0], np.cumsum(L)]).astype(np.int64)
        V = 4
        words = rng.integers(0, V, size=doc_ptr[-1]).astype(np.int32)
        z = rng.integers(0, K, size=doc_ptr[-1]).astype(np.uint16)
        m = O.OracleLDA(6, V, K, 0.3, 0.07).load(doc_ptr, words, 1)
        m.set_z(z)
        expect = _polya_sequence_logprob(doc_ptr, words, z, V, K, 0.3, 0.07) / doc_ptr[-1]
        assert m.loglik() == pytest.approx(expect, rel=1e-12, abs=1e-12)


def test_loglik_k1_dirichlet_multinomial():
    """K = 1: the doc part vanishes and the word part is the Dirichlet-
    multinomial lgΓ(Vβ) − lgΓ(T+Vβ) + Σ_w [lgΓ(n_w+β) − lgΓ(β)]."""
    rng = np.random.default_rng(11)
    L = rng.integers(1, 40, size=30)
    doc_ptr = np.concatenate([[0], np.cumsum(L)]).astype(np.int64)
    V, T, b = 25, int(doc_ptr[-1]), 0.01
    words = rng.integers(0, V, size=T).astype(np.int32)
    m = O.OracleLDA(30, V, 1, 50.0, b).load(doc_ptr, words, 5)
    nw = np.bincount(words, minlength=V)
    closed = gammaln(V * b) - gammaln(T + V * b) + (gammaln(nw + b) - gammaln(b)).sum()
    assert m.loglik() * T == pytest.approx(closed, rel=1e-12)


def test_loglik_relabel_invariance(tiny_corpus, tiny_cfg):
    doc_ptr, words, _ = tiny_corpus
    c = tiny_cfg
    m = O.OracleLDA(c.D, c.V, c.K, c.alpha, c.beta).load(doc_ptr, words, c.seed)
    m.iterate(2)
    ll = m.loglik()
    perm = np.random.default_rng(0).permutation(c.K).astype(np.uint16)
    m.set_z(perm[m.z])
    assert m.loglik() == pytest.approx(ll, rel=1e-12)


def test_loglik_rises_on_tiny(tiny_corpus, tiny_cfg):
    """SURVEY §8(c) convergence pin (tiny config, LDA-generated): LL rises
    strictly at every sweep 1..20 and gains >= 0.5 nat/token."""
    doc_ptr, words, _ = tiny_corpus
    c = tiny_cfg
    m = O.OracleLDA(c.D, c.V, c.K, c.alpha, c.beta).load(doc_ptr, words, c.seed)
    ll = [m.loglik()]
    for _ in range(c.sweeps):
        m.iterate(1)
        ll.append(m.loglik())
        assert m.invariants() == 0
    assert np.all(np.diff(ll) > 0)
    assert ll[-1] - ll[0] >= 0.5
    assert -15.0 <= ll[-1] <= 0.0      # Fig. 8 axis range (L1509-1519)


def test_oracle_omp_sweep_bit_identical():
    """oracle-omp: the SWEEP with documents drawn on all host
    cores must give exactly the single-threaded oracle's z, counts and
    margins -- each draw reads only frozen counts and its own counter-based
    uniform (X3, X9), so the order of the documents cannot matter."""
    from paper_conf_hpdc_xie0lt19_b200 import synth
    cfg = synth.scaled(synth.CONFIGS["nytimes"], 0.0005)          # ~50k tokens
    doc_ptr, words = synth.to_numpy(*synth.generate_config(cfg, "cpu"))[:2]
    K = 64
    a = O.OracleLDA(cfg.D, cfg.V, K, 50.0 / K, 0.01).load(doc_ptr, words, 3)
    b = O.OracleLDA(cfg.D, cfg.V, K, 50.0 / K, 0.01).load(doc_ptr, words, 3)
    for _ in range(3):
        ma = a.iterate(1, margins=True)
        mb = b.iterate(1, margins=True, parallel=True)
        assert np.array_equal(a.z, b.z)
        assert np.array_equal(ma, mb)
        assert np.array_equal(a.n_wk, b.n_wk) and np.array_equal(a.n_k, b.n_k)
        assert np.array_equal(a.n_dk, b.n_dk)
    assert O.omp_threads() >= 1
