"""f3: out-of-HBM streaming, Alg. 1 WorkSchedule2 (PAPER.md
L835-859; §5.1) -- option stream_chunks = M > 1 (-m gpu).

Each rank's documents are cut into M chunks whose token tables, z and θ rows
live in page-locked host memory; every sweep streams each chunk through one of
two device slots (the transfer of chunk m+1 overlapping the sampling of chunk
m, L925-931) while n_wk and the word tables stay resident.  The draws are a
function of the frozen counts and each token's global canonical index only,
so every M must give exactly the resident (M = 1) run: z, n_wk, n_k, θ
bit-identical, LL equal; and M > 1 composes with world > 1.
"""
import numpy as np
import pytest

import lda_testutil as U
from paper_conf_hpdc_xie0lt19_b200 import synth
from test_gpu_multirank import run_ranks, _check_equal_to_one_rank

pytestmark = pytest.mark.gpu


def _nyt():
    cfg = synth.scaled(synth.CONFIGS["nytimes"], 0.01)        # ~1 M tokens
    doc_ptr, words = synth.to_numpy(*synth.generate_config(cfg, "cpu"))[:2]
    return cfg, doc_ptr, words


@pytest.mark.parametrize("K,opts", [
    (1024, dict(stream_chunks=2)),
    (1024, dict(stream_chunks=5, tile_tokens=50_000)),
    (128, dict(stream_chunks=3, sampler=3)),
    (8192, dict(stream_chunks=4)),
])
def test_stream_chunks_equal_resident(K, opts):
    cfg, doc_ptr, words = _nyt()
    a, b = 50.0 / K, 0.01
    ref = U.gpu_model(cfg.D, cfg.V, K, a, b, doc_ptr, words, cfg.seed)
    g = U.gpu_model(cfg.D, cfg.V, K, a, b, doc_ptr, words, cfg.seed, loglik_every=2, **opts)
    assert g.stats()["n_stream_chunks"] == opts["stream_chunks"]
    assert np.array_equal(g.z(), ref.z())
    for sweep in range(4):
        ref.iterate(1)
        g.iterate(1)
        assert np.array_equal(g.z(), ref.z()), sweep
        assert np.array_equal(g.nwk(), ref.nwk())
        assert np.array_equal(g.nk(), ref.nk())
        pr, tr, cr = ref.theta_csr()
        pg, tg, cg = g.theta_csr()
        assert np.array_equal(pr, pg) and np.array_equal(tr, tg) and np.array_equal(cr, cg)
        assert g.loglik() == pytest.approx(ref.loglik(), rel=1e-12)
        assert g.stats()["sum_nnz_tok"] == ref.stats()["sum_nnz_tok"]
    lg = g.loglik_log()                     # the last call was sweep t = 4 (loglik_every = 2)
    assert lg["sweep"].tolist() == [4]
    assert lg["ll_per_token"][0] == pytest.approx(ref.loglik(), rel=1e-12)
    U.check_invariants_gpu(g, doc_ptr, words)


def test_stream_chunks_oracle_lockstep_and_set_z():
    """M = 3 against the oracle in lock step (north_star excuse rule), with
    teacher forcing through lda_set_z on the streamed state."""
    c = synth.CONFIGS["tiny"]
    doc_ptr, words = synth.tiny_numpy()[:2]
    o = U.oracle_for(c.D, c.V, c.K, c.alpha, c.beta, doc_ptr, words, c.seed)
    g = U.gpu_model(c.D, c.V, c.K, c.alpha, c.beta, doc_ptr, words, c.seed, stream_chunks=3, tile_tokens=5_000)
    assert np.array_equal(g.z(), o.z)
    U.check_counts_equal(g, o)
    bad, unexc = U.lockstep(g, o, 6)
    assert unexc == 0 and bad <= U.MAX_EXCUSED_FRAC * c.T * 6
    assert g.loglik() == pytest.approx(o.loglik(), rel=1e-9)
    # more chunks than documents: clamped to one chunk per document at most
    g2 = U.gpu_model(3, c.V, c.K, c.alpha, c.beta, doc_ptr[:4], words[:int(doc_ptr[3])], c.seed, stream_chunks=10)
    g2.iterate(2)
    U.check_invariants_gpu(g2, doc_ptr[:4], words[:int(doc_ptr[3])])


@pytest.mark.parametrize("world,opts", [(2, dict(stream_chunks=3)), (3, dict(stream_chunks=2, sampler=3))])
def test_stream_chunks_with_ranks(world, opts):
    """WorkSchedule2 with G > 1 ranks (C = M x G chunks, L787-793): equal to
    one resident rank bitwise."""
    cfg, doc_ptr, words = _nyt()
    one = run_ranks(1, cfg.D, cfg.V, 1024, doc_ptr, words, 5, 3, {})
    many = run_ranks(world, cfg.D, cfg.V, 1024, doc_ptr, words, 5, 3, opts)
    _check_equal_to_one_rank(one, many, world)


def test_stream_chunks_rejects_sampler0():
    import paper_conf_hpdc_xie0lt19_b200 as L
    c = synth.CONFIGS["tiny"]
    doc_ptr, words = synth.tiny_numpy()[:2]
    with pytest.raises(L.LDAError) as e:
        U.gpu_model(c.D, c.V, c.K, c.alpha, c.beta, doc_ptr, words, c.seed, stream_chunks=2, sampler=0)
    assert e.value.code == L.LDA_EINVAL
