"""The library's world > 1 path on ONE B200 (-m gpu): `world` contexts in one
process, each driven by its own thread and joined into an in-process peer
group (include/lda.h lda_peer_group_*), so every multi-rank step of
lda_load_corpus / lda_iterate / lda_loglik / lda_set_z runs through the
library:

  * token-balanced document partition (lda_partition_docs, X21, L755-759);
  * all-gather of the per-rank word histograms -> canonical bases (X18);
  * per-rank partial recount of n_wk / n_k, then their sum over the ranks
    (Eq. 4; Alg. 1 lines 14-15, L825-827) on the comm stream,
    overlapped with the θ rebuild (§6.2);
  * the LL's doc part summed over the ranks.

SURVEY §8(c) "Multi-GPU" pin: z on G ranks == z on one GPU bitwise (the
canonical index c is global, the counts are globally identical after the
exchange, the prefix order is partition-independent), the allreduced n_wk
equals the 1-GPU n_wk bitwise, and every rank holds the same replica.
"""
import threading

import numpy as np
import pytest

import lda_testutil as U
import paper_conf_hpdc_xie0lt19_b200 as L
from paper_conf_hpdc_xie0lt19_b200 import synth

pytestmark = pytest.mark.gpu


def _corpus(name):
    if name == "tiny":
        c = synth.CONFIGS["tiny"]
        doc_ptr, words = synth.tiny_numpy()[:2]
        return c.D, c.V, doc_ptr, words
    cfg = synth.scaled(synth.CONFIGS["nytimes"], 0.01)        # ~1 M tokens, NYTimes-shaped
    doc_ptr, words = synth.to_numpy(*synth.generate_config(cfg, "cpu"))[:2]
    return cfg.D, cfg.V, doc_ptr, words


def run_ranks(world, D, V, K, doc_ptr, words, seed, sweeps, opts, set_z_at=None, z_force=None):
    """Run `world` ranks in threads; per sweep record every rank's local z
    (document order), n_wk, n_k and the (collective) LL.  Returns
    {rank: [(z, nwk, nk, ll), ...]} with entry 0 the state after load."""
    bounds = L.lda_partition_docs(doc_ptr, world)
    grp = L.PeerGroup(world) if world > 1 else None
    out = {r: [] for r in range(world)}
    errors = []
    a, b = 50.0 / K, 0.01

    def rank_main(r):
        m = None
        try:
            d0, d1 = int(bounds[r]), int(bounds[r + 1])
            t0, t1 = int(doc_ptr[d0]), int(doc_ptr[d1])
            m = L.LDA(D, V, K, a, b, device=0, **opts)
            if grp is not None:
                m.init_peer(grp, r)
            m.load(doc_ptr[d0:d1 + 1] - t0, words[t0:t1], seed, d0, d1)
            out[r].append((m.z(), m.nwk(), m.nk(), m.loglik()))
            for s in range(1, sweeps + 1):
                m.iterate(1)
                if set_z_at == s:
                    m.set_z(z_force[t0:t1])
                out[r].append((m.z(), m.nwk(), m.nk(), m.loglik()))
            st = m.stats()
            assert st["world"] == world
        except Exception as e:          # noqa: BLE001 -- re-raised in the main thread
            errors.append((r, e))
        finally:
            if m is not None:
                m.close()

    th = [threading.Thread(target=rank_main, args=(r,)) for r in range(world)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout=1200)
    if grp is not None:
        grp.close()
    assert not errors, errors
    assert all(not t.is_alive() for t in th), "a rank hung"
    return out


def _check_equal_to_one_rank(one, many, world):
    for s in range(len(one[0])):
        z1, nwk1, nk1, ll1 = one[0][s]
        zg = np.concatenate([many[r][s][0] for r in range(world)])
        assert np.array_equal(zg, z1), f"z differs at sweep {s}"
        for r in range(world):
            _, nwk, nk, ll = many[r][s]
            assert np.array_equal(nwk, nwk1), f"n_wk of rank {r} differs at sweep {s}"
            assert np.array_equal(nk, nk1), f"n_k of rank {r} differs at sweep {s}"
            # the LL's fp64 partial sums are added in another order
            assert ll == pytest.approx(ll1, rel=1e-12, abs=1e-12)
        # replicas identical across ranks (checksums of the exchanged state)
        sums = {int(many[r][s][1].astype(np.int64).sum() * 1_000_003 + many[r][s][1][:, 0].sum())
                for r in range(world)}
        assert len(sums) == 1


@pytest.mark.parametrize("world,corpus,K,opts", [
    (2, "tiny", 16, {}),
    (3, "tiny", 16, dict(sampler=0)),
    (2, "nytimes1pct", 1024, {}),
    (3, "nytimes1pct", 1024, dict(fused_recount=1, tile_tokens=100_000)),
    (2, "nytimes1pct", 128, dict(sampler=3)),
    (4, "nytimes1pct", 1024, dict(sampler=0)),
    (2, "nytimes1pct", 1024, dict(comm_pipeline=1)),
    (3, "nytimes1pct", 1024, dict(comm_pipeline=17, recount_tokens=300)),
])
def test_world_equals_one_gpu_bitwise(world, corpus, K, opts):
    D, V, doc_ptr, words = _corpus(corpus)
    sweeps = 5
    one = run_ranks(1, D, V, K, doc_ptr, words, 7, sweeps, opts)
    many = run_ranks(world, D, V, K, doc_ptr, words, 7, sweeps, opts)
    _check_equal_to_one_rank(one, many, world)


def test_world2_k8192_cta_sampler():
    doc_ptr, words = synth.to_numpy(*synth.generate(300, 400, 40_000, 0.7, 64, 12, "cpu"))[:2]
    one = run_ranks(1, 300, 400, 8192, doc_ptr, words, 9, 2, {})
    many = run_ranks(2, 300, 400, 8192, doc_ptr, words, 9, 2, {})
    _check_equal_to_one_rank(one, many, 2)


def test_world2_tiny_matches_oracle_and_set_z():
    """Two ranks against the oracle (lock step with the north_star excuse
    rule), and lda_set_z as a collective (teacher forcing at sweep 3)."""
    c = synth.CONFIGS["tiny"]
    doc_ptr, words = synth.tiny_numpy()[:2]
    o = U.oracle_for(c.D, c.V, c.K, c.alpha, c.beta, doc_ptr, words, c.seed)
    margins = []
    zs = [o.z.copy()]
    for _ in range(5):
        margins.append(o.iterate(1, margins=True))
        zs.append(o.z.copy())
    # force the oracle's sweep-3 state into the GPU ranks right after their sweep 3
    many = run_ranks(2, c.D, c.V, c.K, doc_ptr, words, c.seed, 5, {}, set_z_at=3, z_force=zs[3])
    for s in range(6):
        zg = np.concatenate([many[r][s][0] for r in range(2)])
        if s == 0:
            assert np.array_equal(zg, zs[0])
            continue
        bad = np.nonzero(zg != zs[s])[0]
        assert (margins[s - 1][bad] < U.MARGIN_EXCUSE).all()
        assert len(bad) <= U.MAX_EXCUSED_FRAC * c.T + 1


def test_nccl_backend_one_rank():
    """The NCCL data plane (one process per GPU) on this one-GPU box: NCCL
    refuses two ranks on one device, so the backend runs end to end with one
    rank -- dlopen of the process's libnccl.so.2, unique id, communicator,
    the in-place int32 / fp64 allreduces and the int64 all-gather the library
    issues, teardown -- and each collective must be the identity."""
    import torch  # noqa: F401  (loads torch's NCCL first, as in bench.py)
    import paper_conf_hpdc_xie0lt19_b200 as L
    msg = L.lda_debug_nccl_selftest(0)
    assert msg.startswith("nccl:"), msg
