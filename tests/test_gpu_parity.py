"""GPU parity: the CUDA path through the C ABI vs the CPU oracle (-m gpu).

Every case feeds both sides the same seeded synthetic corpus.  Tolerances are
the north_star's (BASELINE.json): integer counts bit-exact; per-token z exact
except tokens whose oracle uniform is within 1e-6 of a CDF boundary (< 1e-4
of all tokens); LL/token within 1e-3 relative.
"""
import json
import os

import numpy as np
import pytest

import lda_testutil as U
from oracle import oracle as O
from paper_conf_hpdc_xie0lt19_b200 import synth

pytestmark = pytest.mark.gpu
GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def _corpus(D, V, T, sigma, K_gen, seed):
    return synth.to_numpy(*synth.generate(D, V, T, sigma, K_gen, seed, "cpu"))[:2]


def test_appendix_a_micro_bit_exact():
    g = json.load(open(os.path.join(GOLDEN, "appendix_a_micro.json")))
    words = np.array(sum(g["docs"], []), np.int32)
    doc_ptr = np.cumsum([0] + [len(d) for d in g["docs"]]).astype(np.int64)
    m = U.gpu_model(g["D"], g["V"], g["K"], g["alpha"], g["beta"], doc_ptr, words, g["seed"])
    canon = O.canonical_order(doc_ptr, words, g["V"])
    inv = np.argsort(canon)
    assert m.z()[inv].tolist() == g["init"]["z_canonical"]
    assert m.nwk().tolist() == g["init"]["n_wk"]
    assert m.ndk_dense().tolist() == g["init"]["n_dk"]
    assert m.nk().tolist() == g["init"]["n_k"]
    assert m.loglik() == pytest.approx(g["init"]["ll_per_token"], rel=1e-10)
    for sw in g["sweeps"]:
        m.iterate(1)
        assert m.z()[inv].tolist() == sw["z_canonical"]
        assert m.nwk().tolist() == sw["n_wk"]
        assert m.ndk_dense().tolist() == sw["n_dk"]
        assert m.nk().tolist() == sw["n_k"]
        assert m.loglik() == pytest.approx(sw["ll_per_token"], rel=1e-10)


def test_tiny_config_lockstep_and_ll():
    """BASELINE configs[0]: D=1000, V=500, K=16, 50k tokens, 20 sweeps."""
    c = synth.CONFIGS["tiny"]
    doc_ptr, words = synth.tiny_numpy()[:2]
    o = U.oracle_for(c.D, c.V, c.K, c.alpha, c.beta, doc_ptr, words, c.seed)
    g = U.gpu_model(c.D, c.V, c.K, c.alpha, c.beta, doc_ptr, words, c.seed)
    assert np.array_equal(g.z(), o.z)          # init is integer: bit-exact
    U.check_counts_equal(g, o)
    assert g.loglik() == pytest.approx(o.loglik(), rel=1e-9)
    bad, unexc = U.lockstep(g, o, c.sweeps, teacher_force=True)
    assert unexc == 0
    assert bad <= U.MAX_EXCUSED_FRAC * c.T * c.sweeps
    assert g.loglik() == pytest.approx(o.loglik(), rel=U.LL_RTOL)


def test_tiny_config_free_running_ll_after_100():
    """north_star: per-token LL after 100 iterations within 1e-3 relative."""
    c = synth.CONFIGS["tiny"]
    doc_ptr, words = synth.tiny_numpy()[:2]
    o = U.oracle_for(c.D, c.V, c.K, c.alpha, c.beta, doc_ptr, words, c.seed)
    g = U.gpu_model(c.D, c.V, c.K, c.alpha, c.beta, doc_ptr, words, c.seed)
    o.iterate(100)
    g.iterate(100)
    llo, llg = o.loglik(), g.loglik()
    assert llg == pytest.approx(llo, rel=U.LL_RTOL)
    U.check_invariants_gpu(g, doc_ptr, words)
    # the chains stayed identical (fp64 probabilities; SURVEY §7 "LL@100")
    assert np.mean(g.z() != o.z) < 1e-3


def test_nytimes_1pct_ll_after_100_parity():
    """north_star: LL/token after 100 iterations within 1e-3 relative of the
    oracle's, at a real size: a NYTimes-shaped 1 % corpus (~1 M tokens,
    K = 1024, the defaults), 100 free-running sweeps on each side.  The oracle
    runs as oracle-omp (bit-identical to the single-threaded oracle, pinned in
    test_oracle_pins.py) on all host cores.  The two chains are expected to
    stay identical (a boundary flip needs the uniform within ~1e-13 of a CDF
    boundary: ~1e-3 expected flips in 10^8 draws)."""
    cfg = synth.scaled(synth.CONFIGS["nytimes"], 0.01)
    doc_ptr, words = synth.to_numpy(*synth.generate_config(cfg, "cpu"))[:2]
    o = U.oracle_for(cfg.D, cfg.V, cfg.K, cfg.alpha, cfg.beta, doc_ptr, words, cfg.seed)
    g = U.gpu_model(cfg.D, cfg.V, cfg.K, cfg.alpha, cfg.beta, doc_ptr, words, cfg.seed, loglik_every=10)
    g.iterate(100)
    o.iterate(100, parallel=True)
    llo, llg = o.loglik(), g.loglik()
    same = float(np.mean(g.z() == o.z))
    print(f"NYTimes 1%: LL@100 gpu {llg:.8f} oracle {llo:.8f} (rel {abs(llg - llo) / abs(llo):.2e}); "
          f"z identical {same:.6f}; oracle-omp threads {O.omp_threads()}")
    assert llg == pytest.approx(llo, rel=U.LL_RTOL)
    assert same > 0.999
    U.check_invariants_gpu(g, doc_ptr, words)
    # the LL log of the same call (option loglik_every): sweeps 10, 20, ..., 100, rising overall
    lg = g.loglik_log()
    assert lg["sweep"].tolist() == list(range(10, 101, 10))
    assert lg["ll_per_token"][-1] == pytest.approx(llg, rel=1e-12)
    assert lg["ll_per_token"][-1] > lg["ll_per_token"][0]


@pytest.mark.parametrize("sampler", [2, 3, 0])
@pytest.mark.parametrize("K", [1, 2, 37, 128, 1024])
def test_k_variants_lockstep(K, sampler):
    """Every sampler (2 = tile sampler, the default; 3 = its CTA-shared-table
    form for large K; 0 = lane per token) against the oracle."""
    doc_ptr, words = _corpus(600, 700, 60_000, 0.7, 16, 11)
    a, b = 50.0 / K, 0.01
    o = U.oracle_for(600, 700, K, a, b, doc_ptr, words, 5)
    g = U.gpu_model(600, 700, K, a, b, doc_ptr, words, 5, sampler=sampler)
    assert np.array_equal(g.z(), o.z)
    U.check_counts_equal(g, o)
    bad, unexc = U.lockstep(g, o, 3)
    assert unexc == 0 and bad <= U.MAX_EXCUSED_FRAC * 60_000 * 3
    assert g.loglik() == pytest.approx(o.loglik(), rel=1e-9)


@pytest.mark.parametrize("opts", [dict(sampler=-1), dict(sampler=2), dict(sampler=0),
                                  dict(sampler=3, fused_recount=1)])
def test_k8192_small(opts):
    """K = 8192: the default (auto -> the CTA tile sampler), the per-warp tile
    sampler, the lane-per-token sampler, and the CTA sampler with the fused
    recount (n_k by global reductions, the GNK path)."""
    doc_ptr, words = _corpus(300, 400, 40_000, 0.7, 64, 12)
    K = 8192
    o = U.oracle_for(300, 400, K, 50.0 / K, 0.01, doc_ptr, words, 9)
    g = U.gpu_model(300, 400, K, 50.0 / K, 0.01, doc_ptr, words, 9, **opts)
    bad, unexc = U.lockstep(g, o, 2)
    assert unexc == 0


@pytest.mark.parametrize("K,opts", [(20000, {}), (65536, {}), (30000, dict(exclude_self=1))])
def test_wide_k_lockstep(K, opts):
    """16384 < K <= 65536 (u16 topic ids, L1239-1243): wide θ entries
    (topic << 16 | count), K-length histograms in global scratch, the
    lane-per-token sampler -- against the oracle in lock step."""
    doc_ptr, words = _corpus(60, 150, 6_000, 0.7, 16, 41)
    a, b = 50.0 / K, 0.01
    excl = opts.get("exclude_self", 0)
    o = U.oracle_for(60, 150, K, a, b, doc_ptr, words, 4)
    g = U.gpu_model(60, 150, K, a, b, doc_ptr, words, 4, **opts)
    assert g.stats()["sampler"] == 0
    assert np.array_equal(g.z(), o.z)
    U.check_counts_equal(g, o)
    bad, unexc = U.lockstep(g, o, 3, exclude_self=excl)
    assert unexc == 0
    assert g.loglik() == pytest.approx(o.loglik(), rel=1e-9)
    U.check_invariants_gpu(g, doc_ptr, words)


def test_nytimes_shaped_midsize_many_chunks():
    """A downscaled NYTimes-shaped corpus at K=1024 that spans many sampler
    chunks, split words and ragged tails; options that only change the work
    decomposition must give bit-identical results."""
    cfg = synth.scaled(synth.CONFIGS["nytimes"], 0.002)       # ~200k tokens, V=101636
    doc_ptr, words = synth.to_numpy(*synth.generate_config(cfg, "cpu"))[:2]
    o = U.oracle_for(cfg.D, cfg.V, cfg.K, cfg.alpha, cfg.beta, doc_ptr, words, cfg.seed)
    g = U.gpu_model(cfg.D, cfg.V, cfg.K, cfg.alpha, cfg.beta, doc_ptr, words, cfg.seed)
    bad, unexc = U.lockstep(g, o, 3)
    assert unexc == 0 and bad <= U.MAX_EXCUSED_FRAC * cfg.T * 3
    z_ref = g.z()
    for opts in [dict(chunk_tokens=100, recount_tokens=300), dict(tile_tokens=30_000),
                 dict(chunk_tokens=33, tile_tokens=7_000, recount_tokens=256, threads=3),
                 dict(tile_tokens=0), dict(tile_tokens=20_000, fused_recount=1),
                 dict(sampler=3, tile_tokens=30_000)]:
        h = U.gpu_model(cfg.D, cfg.V, cfg.K, cfg.alpha, cfg.beta, doc_ptr, words, cfg.seed, **opts)
        h.iterate(3)
        assert np.array_equal(h.z(), z_ref), opts
        assert np.array_equal(h.nwk(), g.nwk())
    # the other samplers on the same corpus
    for opts in [dict(sampler=3), dict(sampler=0), dict(sampler=0, chunk_tokens=100)]:
        h = U.gpu_model(cfg.D, cfg.V, cfg.K, cfg.alpha, cfg.beta, doc_ptr, words, cfg.seed, **opts)
        o = U.oracle_for(cfg.D, cfg.V, cfg.K, cfg.alpha, cfg.beta, doc_ptr, words, cfg.seed)
        bad, unexc = U.lockstep(h, o, 3)
        assert unexc == 0 and bad <= U.MAX_EXCUSED_FRAC * cfg.T * 3, opts


def test_exclude_self_lockstep():
    doc_ptr, words = _corpus(500, 300, 30_000, 0.5, 16, 13)
    K = 24
    o = U.oracle_for(500, 300, K, 50.0 / K, 0.01, doc_ptr, words, 3)
    g = U.gpu_model(500, 300, K, 50.0 / K, 0.01, doc_ptr, words, 3, exclude_self=1)
    bad, unexc = U.lockstep(g, o, 3, exclude_self=1)
    assert unexc == 0 and bad <= U.MAX_EXCUSED_FRAC * 30_000 * 3


@pytest.mark.parametrize("sampler,extra", [(2, {}), (3, {}), (0, {}), (2, dict(tile_tokens=5_000))])
def test_edge_cases(sampler, extra):
    rng = np.random.default_rng(4)
    # empty docs, single-token docs, a 65535-token doc, absent words, D=1
    L_d = np.array([0, 1, 0, 5, 65535, 1, 0, 3] + list(rng.integers(0, 20, 50)), np.int64)
    doc_ptr = np.concatenate([[0], np.cumsum(L_d)]).astype(np.int64)
    V = 300
    words = rng.integers(0, V // 2, size=doc_ptr[-1]).astype(np.int32)   # words >= 150 absent
    D, K = len(L_d), 40
    o = U.oracle_for(D, V, K, 0.3, 0.02, doc_ptr, words, 77)
    g = U.gpu_model(D, V, K, 0.3, 0.02, doc_ptr, words, 77, chunk_tokens=64, sampler=sampler, **extra)
    assert np.array_equal(g.z(), o.z)
    U.check_counts_equal(g, o)
    bad, unexc = U.lockstep(g, o, 3)
    assert unexc == 0
    U.check_invariants_gpu(g, doc_ptr, words)
    assert g.loglik() == pytest.approx(o.loglik(), rel=1e-9)
    # D = 1, a single token
    o1 = U.oracle_for(1, 1, 3, 0.5, 0.1, np.array([0, 1]), np.array([0], np.int32), 1)
    g1 = U.gpu_model(1, 1, 3, 0.5, 0.1, np.array([0, 1]), np.array([0], np.int32), 1, sampler=sampler)
    U.lockstep(g1, o1, 5)


def test_tile_sampler_decomposition_and_fallback_rate():
    """The tile sampler (default) on a ~1 M-token NYTimes-shaped corpus: the
    draws do not depend on the tile / item decomposition, match the fp64
    lane-per-token sampler except within fp64 rounding of a CDF boundary,
    and the fp32 filter sends only a small fraction of tokens to the exact
    fp64 redraw."""
    cfg = synth.scaled(synth.CONFIGS["nytimes"], 0.01)
    doc_ptr, words = synth.to_numpy(*synth.generate_config(cfg, "cpu"))[:2]
    ga = U.gpu_model(cfg.D, cfg.V, cfg.K, cfg.alpha, cfg.beta, doc_ptr, words, cfg.seed, tile_tokens=100_000)
    gb = U.gpu_model(cfg.D, cfg.V, cfg.K, cfg.alpha, cfg.beta, doc_ptr, words, cfg.seed, tile_tokens=0,
                     chunk_tokens=77)
    gc = U.gpu_model(cfg.D, cfg.V, cfg.K, cfg.alpha, cfg.beta, doc_ptr, words, cfg.seed, tile_tokens=300_000,
                     sampler=3)     # CTA-shared tables: same arithmetic, other batches
    gd = U.gpu_model(cfg.D, cfg.V, cfg.K, cfg.alpha, cfg.beta, doc_ptr, words, cfg.seed, tile_tokens=100_000,
                     fused_recount=1)   # n_wk / n_k by the sampler's own reductions instead of the recount kernel
    g0 = U.gpu_model(cfg.D, cfg.V, cfg.K, cfg.alpha, cfg.beta, doc_ptr, words, cfg.seed, sampler=0)
    n_exact = 0
    for _ in range(6):
        ga.iterate(1)
        n_exact += ga.stats()["n_exact_redraws"]
        gb.iterate(1)
        gc.iterate(1)
        gd.iterate(1)
        g0.iterate(1)
        za = ga.z()
        assert np.array_equal(za, gb.z())
        assert np.array_equal(za, gc.z())
        assert np.array_equal(za, gd.z())
        assert np.array_equal(ga.nwk(), gd.nwk()) and np.array_equal(ga.nk(), gd.nk())
        diff = np.count_nonzero(za != g0.z())
        assert diff <= 1e-6 * cfg.T + 2
        if diff:                       # keep the chains in lock step
            g0.set_z(za)
    assert n_exact <= 2e-3 * cfg.T * 6, n_exact


@pytest.mark.parametrize("sampler", [2, 3])
@pytest.mark.parametrize("K", [37, 1024, 8192])
def test_tile_sampler_exact_redraw_path(K, sampler):
    """Inflating the tile sampler's certification bounds (certify_slack) sends
    most tokens through the warp-collective fp64 redraw; the chains must still
    match the oracle in lock step (the redraw is the exact path, not a
    different sampler) and the filtered run."""
    doc_ptr, words = _corpus(800, 900, 80_000, 0.7, 16, 31)
    a, b = 50.0 / K, 0.01
    o = U.oracle_for(800, 900, K, a, b, doc_ptr, words, 6)
    g = U.gpu_model(800, 900, K, a, b, doc_ptr, words, 6, certify_slack=1 << 20, tile_tokens=20_000,
                    sampler=sampler)
    h = U.gpu_model(800, 900, K, a, b, doc_ptr, words, 6, tile_tokens=20_000, sampler=sampler)
    n_exact = 0
    for _ in range(3):
        margins = o.iterate(1, margins=True)
        g.iterate(1)
        h.iterate(1)
        n_exact += g.stats()["n_exact_redraws"]
        zg = g.z()
        bad = np.nonzero(zg != o.z)[0]
        assert (margins[bad] < U.MARGIN_EXCUSE).all()
        assert np.count_nonzero(zg != h.z()) <= 2
        if len(bad):
            g.set_z(o.z)
            h.set_z(o.z)
    assert n_exact > 0.3 * 80_000 * 3, n_exact
    U.check_counts_equal(g, o)


def test_set_z_and_determinism():
    doc_ptr, words = _corpus(400, 500, 40_000, 0.5, 16, 21)
    K = 64
    g1 = U.gpu_model(400, 500, K, 50.0 / K, 0.01, doc_ptr, words, 8)
    g2 = U.gpu_model(400, 500, K, 50.0 / K, 0.01, doc_ptr, words, 8)
    g1.iterate(4)
    g2.iterate(4)
    assert np.array_equal(g1.z(), g2.z())            # two runs, identical z
    # checkpoint/resume: z + sweep counter + seed are the whole state
    z = g1.z()
    g3 = U.gpu_model(400, 500, K, 50.0 / K, 0.01, doc_ptr, words, 8)
    g3.iterate(4)            # advance the counter to the same t ...
    g3.set_z(z)              # ... and overwrite the state
    g1.iterate(2)
    g3.iterate(2)
    assert np.array_equal(g1.z(), g3.z())
    assert np.array_equal(g1.nwk(), g3.nwk())


def test_convergence_harness_ll_rises():
    """the LL-vs-time harness on the tiny config — time
    accumulates and the per-token LL rises from the random initialisation."""
    import importlib.util
    spec = importlib.util.spec_from_file_location(
        "convergence", os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                    "tools", "convergence.py"))
    conv = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(conv)
    pts = conv.run("tiny", sweeps=20, every=5, device_index=0, quiet=True)
    assert [p["sweep"] for p in pts] == [0, 5, 10, 15, 20]
    assert all(b["ms"] > a["ms"] for a, b in zip(pts, pts[1:]))
    assert pts[-1]["ll_per_token"] > pts[0]["ll_per_token"] + 0.05


@pytest.mark.parametrize("tile_tokens", [0, 500])
def test_invalid_word_ids_rejected_on_device(tile_tokens):
    """With one rank and a tile sampler the word ids are validated by the
    layout's own count pass (no separate pass over the words): an id outside
    [0, V) must still fail with LDA_EINVAL -- with one tile and with many
    (the thread-per-tile pass)."""
    import paper_conf_hpdc_xie0lt19_b200 as L
    doc_ptr, words = _corpus(400, 300, 30_000, 0.5, 16, 3)
    for bad in (300, -1, 1 << 20):
        w = words.copy()
        w[len(w) // 2] = bad
        with pytest.raises(L.LDAError) as e:
            U.gpu_model(400, 300, 16, 0.5, 0.01, doc_ptr, w, 1, tile_tokens=tile_tokens)
        assert e.value.code == L.LDA_EINVAL, e.value
    g = U.gpu_model(400, 300, 16, 0.5, 0.01, doc_ptr, words, 1, tile_tokens=tile_tokens)
    U.check_invariants_gpu(g, doc_ptr, words)


@pytest.mark.parametrize("n,bits", [(1, 1), (4095, 7), (4097, 23), (300_000, 17), (1_000_003, 23), (70_000, 32)])
def test_device_radix_sort_stable(n, bits):
    """The device radix sort the load uses for the doc-word map: equal to a
    stable sort (numpy mergesort) on the low `bits` key bits, values carried."""
    import paper_conf_hpdc_xie0lt19_b200 as L
    rng = np.random.default_rng(n + bits)
    # Zipf-like keys: long runs of equal keys test the stability
    keys = (rng.zipf(1.3, n) % (1 << min(bits, 31))).astype(np.uint32)
    if bits == 32:
        keys = rng.integers(0, 1 << 32, n, dtype=np.uint64).astype(np.uint32)
    vals = np.arange(n, dtype=np.uint32)
    ok, ov = L.lda_debug_radix_sort(keys, vals, bits)
    order = np.argsort(keys, kind="stable")
    assert np.array_equal(ok, keys[order]) and np.array_equal(ov, vals[order])


@pytest.mark.parametrize("opts", [dict(), dict(tile_tokens=20_000), dict(fused_recount=1, tile_tokens=50_000)])
def test_k8192_sparse_word_rows_bit_identical(opts):
    """f2 (SparseLDA's split p* = β/(n_k+Vβ) + n_wk/(n_k+Vβ), ref [32], L999):
    the large-K sampler rebuilds a rare word's p32 row in shared memory from
    the shared smoothing row patched at the word's nonzero topics, instead of
    copying an O(K) row the table kernel wrote.  The tables are bit-identical,
    so the draws must be too -- for every threshold (none, the default K/4,
    every word), over several sweeps (buffers switch between dense and sparse
    words and are patched / restored) -- and the chain matches the oracle."""
    cfg = synth.scaled(synth.CONFIGS["nytimes_k8192"], 0.003)
    doc_ptr, words = synth.to_numpy(*synth.generate_config(cfg, "cpu"))[:2]
    K = cfg.K
    runs = {thr: U.gpu_model(cfg.D, cfg.V, K, cfg.alpha, cfg.beta, doc_ptr, words, cfg.seed, sparse_words=thr,
                             **opts) for thr in (0, -1, 1 << 40)}
    assert runs[0].stats()["n_sparse_words"] == 0
    nsp = runs[-1].stats()["n_sparse_words"]
    wc = np.bincount(words, minlength=cfg.V)
    assert nsp == int(((wc > 0) & (wc <= K // 4)).sum()) and nsp > 0
    assert runs[1 << 40].stats()["n_sparse_words"] == int((wc > 0).sum())
    o = U.oracle_for(cfg.D, cfg.V, K, cfg.alpha, cfg.beta, doc_ptr, words, cfg.seed)
    for _ in range(3):
        margins = o.iterate(1, margins=True)
        for g in runs.values():
            g.iterate(1)
        z0 = runs[0].z()
        for thr, g in runs.items():
            assert np.array_equal(g.z(), z0), thr
            assert np.array_equal(g.nwk(), runs[0].nwk()), thr
        bad = np.nonzero(z0 != o.z)[0]
        assert (margins[bad] < U.MARGIN_EXCUSE).all()
        if len(bad):
            for g in runs.values():
                g.set_z(o.z)
    U.check_counts_equal(runs[-1], o)
