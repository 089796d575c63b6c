"""The C-ABI library on a CPU-only host (-m "not gpu"): it loads, exports every
symbol include/lda.h declares, validates its arguments before touching the
device, partitions documents by tokens (X21), and fails loudly (LDA_ECUDA)
rather than falling back when there is no GPU."""
import os
import re

import numpy as np
import pytest

import paper_conf_hpdc_xie0lt19_b200 as L

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _header_symbols():
    src = open(os.path.join(ROOT, "include", "lda.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return set(re.findall(r"\b(lda_[a-z_]+)\s*\(", src))


def test_library_exports_every_declared_symbol():
    lib = L.lib()
    declared = _header_symbols()
    assert declared == set(L.ABI_SYMBOLS)
    for name in declared:
        assert hasattr(lib, name), name
    assert "sm_100a" in L.lda_version()


def test_create_validation():
    ok = L.lda_create(10, 5, 16, 0.1, 0.01)
    L.lda_destroy(ok)
    for args in [(0, 5, 16, 0.1, 0.01), (10, 0, 16, 0.1, 0.01), (10, 5, 0, 0.1, 0.01),
                 (10, 5, 65537, 0.1, 0.01), (10, 5, 16, 0.0, 0.01), (10, 5, 16, 0.1, -1.0),
                 (10, 5, 16, float("nan"), 0.01), (10, 5, 16, 0.1, float("inf"))]:
        with pytest.raises(L.LDAError) as e:
            L.lda_create(*args)
        assert e.value.code == L.LDA_EINVAL
    # u16 topic ids: K up to 65536 (L1239-1243)
    for K in (16384, 16385, 65536):
        L.lda_destroy(L.lda_create(1, 1, K, 1.0, 1.0))


def test_options_validation():
    ctx = L.lda_create(10, 5, 16, 0.1, 0.01)
    try:
        L.lda_set_option(ctx, "exclude_self", 1)
        L.lda_set_option(ctx, "chunk_tokens", 64)
        L.lda_set_option(ctx, "tile_tokens", 0)
        L.lda_set_option(ctx, "tile_tokens", -1)
        L.lda_set_option(ctx, "loglik_every", 5)
        for v in (-1, 0, 4096):
            L.lda_set_option(ctx, "sparse_words", v)   # f2: -1 = K/4, 0 = off, n = threshold
        for key, val in [("exclude_self", 2), ("chunk_tokens", 1), ("nonsense", 1), ("device", -1),
                         ("sampler", 1), ("tile_tokens", -2), ("loglik_every", -1), ("theta_mode", 1),
                         ("filter32", 1), ("sparse_words", -2)]:
            with pytest.raises(L.LDAError) as e:
                L.lda_set_option(ctx, key, val)
            assert e.value.code == L.LDA_EINVAL
        # calls that need a corpus
        for f in (lambda: L.lda_iterate(ctx, 1), lambda: L.lda_loglik(ctx),
                  lambda: L.lda_get_stream(ctx)):
            with pytest.raises(L.LDAError) as e:
                f()
            assert e.value.code == L.LDA_ESTATE
    finally:
        L.lda_destroy(ctx)


def test_partition_docs_token_balanced():
    rng = np.random.default_rng(1)
    for D, world in [(1, 1), (5, 8), (100, 3), (1000, 8), (7, 2)]:
        L_d = rng.integers(0, 50, size=D)
        doc_ptr = np.concatenate([[0], np.cumsum(L_d)]).astype(np.int64)
        T = int(doc_ptr[-1])
        b = L.lda_partition_docs(doc_ptr, world)
        assert b[0] == 0 and b[-1] == D and np.all(np.diff(b) >= 0)
        for g in range(1, world):
            target = -(-g * T // world)   # ceil(g T / world)
            expect = int(np.argmax(doc_ptr >= target)) if (doc_ptr >= target).any() else D
            assert b[g] == max(expect, b[g - 1])
    with pytest.raises(L.LDAError):
        L.lda_partition_docs(np.array([0, 3, 2], np.int64), 2)


def test_load_validation_before_device():
    doc_ptr = np.array([0, 3, 5], np.int64)
    words = np.array([0, 1, 2, 3, 4], np.int32)
    cases = [
        (dict(doc_ptr=np.array([1, 3, 5], np.int64)), L.LDA_EINVAL),            # doc_ptr[0] != 0
        (dict(doc_ptr=np.array([0, 3, 2], np.int64)), L.LDA_EINVAL),            # decreasing
        (dict(words=np.array([0, 1, 2, 3, 5], np.int32)), L.LDA_EINVAL),        # id >= V
        (dict(words=np.array([0, -1, 2, 3, 4], np.int32)), L.LDA_EINVAL),       # id < 0
        (dict(doc_end=3), L.LDA_EINVAL),                                         # range > D
    ]
    for over, code in cases:
        ctx = L.lda_create(2, 5, 8, 0.1, 0.01)
        try:
            kw = dict(doc_begin=0, doc_end=2, doc_ptr=doc_ptr, words=words, seed=1)
            kw.update(over)
            with pytest.raises(L.LDAError) as e:
                L.lda_load_corpus(ctx, **kw)
            assert e.value.code == code, (over, e.value)
        finally:
            L.lda_destroy(ctx)
    # a document longer than 65535 tokens (uint16 θ counts) -> LDA_ERANGE
    ctx = L.lda_create(1, 2, 8, 0.1, 0.01)
    try:
        with pytest.raises(L.LDAError) as e:
            L.lda_load_corpus(ctx, 0, 1, np.array([0, 65536], np.int64), np.zeros(65536, np.int32), 1)
        assert e.value.code == L.LDA_ERANGE
    finally:
        L.lda_destroy(ctx)


def test_no_gpu_fails_loudly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    ctx = L.lda_create(2, 5, 8, 0.1, 0.01)
    try:
        with pytest.raises(L.LDAError) as e:
            L.lda_load_corpus(ctx, 0, 2, np.array([0, 3, 5], np.int64), np.arange(5, dtype=np.int32), 1)
        assert e.value.code == L.LDA_ECUDA
        # sticky: the context stays failed
        with pytest.raises(L.LDAError) as e2:
            L.lda_iterate(ctx, 1)
        assert e2.value.code == L.LDA_ECUDA
    finally:
        L.lda_destroy(ctx)


def _corpus(D, V, seed, max_len=40, empty=True):
    rng = np.random.default_rng(seed)
    L_d = rng.integers(0 if empty else 1, max_len, size=D)
    doc_ptr = np.concatenate([[0], np.cumsum(L_d)]).astype(np.int64)
    # Zipf-like word frequencies: heavy heads, many rare words (tail tile)
    p = 1.0 / np.arange(1, V + 1)
    words = rng.choice(V, size=int(doc_ptr[-1]), p=p / p.sum()).astype(np.int32)
    return doc_ptr, words


@pytest.mark.parametrize("sampler", [0, 2, 3])
@pytest.mark.parametrize("tile_tokens,chunk_tokens,tail", [(0, 4096, 64), (900, 4096, 64), (700, 33, 8),
                                                            (500, 7, 1000), (300, 64, 0)])
def test_layout_invariants(sampler, tile_tokens, chunk_tokens, tail):
    """The host token layout (no GPU): doc_map a permutation, rows per token,
    runs per word, and -- for the tile samplers -- canonical ranks
    crank0 + j for every item token (checked against brute force)."""
    doc_ptr, words = _corpus(400, 300, 5)
    st = L.lda_layout_selfcheck(doc_ptr, words, 300, 24, sampler=sampler, tile_tokens=tile_tokens,
                                chunk_tokens=chunk_tokens, tail_per_tile=tail)
    if sampler >= 2 and tile_tokens and tail:
        assert st["tiles"] >= 2 and st["tail_words"] > 0      # the tail tile is exercised
    assert st["items"] > 0 and st["runs"] > 0


@pytest.mark.parametrize("sampler", [0, 2])
def test_layout_invariants_multithreaded_tiles(sampler):
    """Tiles of >= 2^16 tokens are split over the host threads (per-part
    counts, per-word bases computed in parallel over word ranges): the same
    invariants as above."""
    doc_ptr, words = _corpus(5000, 3000, 9, max_len=80)
    st = L.lda_layout_selfcheck(doc_ptr, words, 3000, 24, sampler=sampler, tile_tokens=90_000,
                                chunk_tokens=512, tail_per_tile=8)
    assert st["tiles"] >= 3 and st["items"] > 0 and st["runs"] > 0


def test_layout_selfcheck_rejects_bad_input():
    doc_ptr, words = _corpus(10, 20, 1)
    bad = words.copy()
    bad[0] = 20                                               # word id >= V
    with pytest.raises(L.LDAError):
        L.lda_layout_selfcheck(doc_ptr, bad, 20, 4)


def test_peer_group_host_validation():
    """In-process peer group (include/lda.h): handle life cycle and join
    validation, no device needed."""
    with pytest.raises(L.LDAError) as e:
        L.lda_peer_group_create(0)
    assert e.value.code == L.LDA_EINVAL
    with pytest.raises(L.LDAError):
        L.lda_peer_group_create(17)
    g = L.PeerGroup(2)
    a = L.lda_create(10, 5, 16, 0.1, 0.01)
    b = L.lda_create(10, 5, 16, 0.1, 0.01)
    c = L.lda_create(10, 5, 16, 0.1, 0.01)
    try:
        L.lda_init_peer(a, g.h, 0)
        for ctx, rank in [(b, 0), (b, 2), (b, -1)]:          # duplicate / out of range
            with pytest.raises(L.LDAError) as e:
                L.lda_init_peer(ctx, g.h, rank)
            assert e.value.code == L.LDA_EINVAL
        L.lda_init_peer(b, g.h, 1)
        with pytest.raises(L.LDAError) as e:                  # a context joins once
            L.lda_init_peer(a, g.h, 1)
        assert e.value.code == L.LDA_ESTATE
        g.close()                                             # contexts keep the group alive
        L.lda_set_option(c, "threads", 2)
    finally:
        for ctx in (a, b, c):
            L.lda_destroy(ctx)


def test_python_binding_checks_buffer_lengths():
    """The ctypes binding refuses short buffers before the C side could read
    or write past them (argument marshalling only)."""
    ctx = L.lda_create(2, 5, 8, 0.1, 0.01)
    try:
        with pytest.raises(L.LDAError) as e:                  # doc_ptr too short for [0, 2)
            L.lda_load_corpus(ctx, 0, 2, np.array([0, 3], np.int64), np.arange(3, dtype=np.int32), 1)
        assert e.value.code == L.LDA_EINVAL
        with pytest.raises(L.LDAError) as e:                  # fewer words than doc_ptr[-1]
            L.lda_load_corpus(ctx, 0, 2, np.array([0, 3, 5], np.int64), np.arange(4, dtype=np.int32), 1)
        assert e.value.code == L.LDA_EINVAL
        with pytest.raises(L.LDAError) as e:
            L.lda_set_z(ctx, np.zeros(3, np.uint16), T=5)
        assert e.value.code == L.LDA_EINVAL
        with pytest.raises(L.LDAError) as e:
            L.lda_get_counts(ctx, n_wk=np.zeros(39, np.int32), shape=(5, 8, 2, 5))
        assert e.value.code == L.LDA_EINVAL
    finally:
        L.lda_destroy(ctx)


@pytest.mark.parametrize("sampler", [2, 3])
def test_layout_invariants_many_tiles(sampler):
    """At least twice as many tiles as host threads (PubMed shape: 54 tiles):
    the host pass runs one thread per tile (counts, run ranks, scatter);
    the same brute-force invariants must hold."""
    import os
    doc_ptr, words = _corpus(6000, 3000, 17, max_len=40)
    tiles_wanted = 2 * (os.cpu_count() or 8) + 3
    tile_tokens = max(50, int(doc_ptr[-1]) // tiles_wanted)
    st = L.lda_layout_selfcheck(doc_ptr, words, 3000, 24, sampler=sampler, tile_tokens=tile_tokens,
                                chunk_tokens=64, tail_per_tile=8)
    assert st["tiles"] >= tiles_wanted and st["tail_words"] > 0
