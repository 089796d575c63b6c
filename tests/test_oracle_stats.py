"""Statistical pins of the oracle's sampler on micro-corpora (-m "not gpu").

These fix the *distribution* the oracle draws from against closed forms:
  * one sweep from a fixed state: each token's law is Eq. 1 (PAPER.md
    L399-409), with the token's own assignment kept in the counts
    (exclude_self = 0, reading X2) -- and the other convention is rejected;
  * SWEEP chains are pairwise independent across tokens within a sweep;
  * SEQUENTIAL mode (textbook CGS) converges to the exact posterior p(z|w),
    enumerated over all K^N states;
  * SWEEP mode (the paper's synchronous iteration, L415-421, X3) converges
    to the exact stationary law of its own K^N x K^N transition matrix, and
    that law is NOT the posterior (so the GPU is never tested against it).
They are blind to mapping conventions (bin order, uniform mapping); those
are pinned by the golden vectors in test_oracle_pins.py.
"""
import itertools

import numpy as np
import pytest
from scipy.special import gammaln
from scipy.stats import chi2, chisquare

from oracle import oracle as O

ALPHA, BETA = 0.5, 0.1
P_CUT = 1e-3   # per-test significance (Bonferroni-adjusted where many)


def _corpus(docs):
    words = np.array(sum(docs, []), np.int32)
    doc_ptr = np.cumsum([0] + [len(d) for d in docs]).astype(np.int64)
    return doc_ptr, words


MICRO8 = [[0, 1, 1, 2], [2, 2, 0, 1]]          # SURVEY §8(d) micro-corpus, V = 3
MICRO5 = [[0, 1, 1], [2, 0]]


def _counts(doc_ptr, words, z, V, K):
    D = len(doc_ptr) - 1
    d = np.repeat(np.arange(D), np.diff(doc_ptr))
    nwk = np.zeros((V, K)); np.add.at(nwk, (words, z), 1)
    ndk = np.zeros((D, K)); np.add.at(ndk, (d, z), 1)
    return nwk, ndk, nwk.sum(0), d


def _eq1(doc_ptr, words, z, V, K, exclude_self):
    """Per-token law of one synchronous sweep, Eq. 1 in closed form."""
    nwk, ndk, nk, d = _counts(doc_ptr, words, z, V, K)
    P = np.empty((len(words), K))
    for i in range(len(words)):
        own = np.zeros(K)
        if exclude_self:
            own[z[i]] = 1
        p = (ndk[d[i]] - own + ALPHA) * (nwk[words[i]] - own + BETA) / (nk - own + V * BETA)
        P[i] = p / p.sum()
    return P


def _pooled_chisq(obs, exp):
    """Chi-square p-value after pooling expected counts < 5 into one bin."""
    obs = np.asarray(obs, float); exp = np.asarray(exp, float)
    small = exp < 5
    o = np.concatenate([obs[~small], [obs[small].sum()]]) if small.any() else obs
    e = np.concatenate([exp[~small], [exp[small].sum()]]) if small.any() else exp
    keep = e > 0
    o, e = o[keep], e[keep]
    stat = ((o - e) ** 2 / e).sum()
    return chi2.sf(stat, len(o) - 1)


# --------------------------------------------------------------------------

@pytest.mark.parametrize("exclude_self", [0, 1])
def test_one_sweep_matches_eq1(exclude_self):
    V, K = 3, 3
    doc_ptr, words = _corpus(MICRO8)
    z0 = np.array([1, 2, 0, 0, 2, 1, 0, 1], np.uint16)      # a fixed state
    n = 100_000
    zf = O.run_chains(doc_ptr, words, V, K, ALPHA, BETA, seed0=1000, n_chains=n,
                      n_sweeps=1, mode="sweep", exclude_self=exclude_self, z_start=z0)
    right = _eq1(doc_ptr, words, z0, V, K, exclude_self)
    wrong = _eq1(doc_ptr, words, z0, V, K, 1 - exclude_self)
    rejected_wrong = 0
    for i in range(len(words)):
        obs = np.bincount(zf[:, i], minlength=K)
        assert chisquare(obs, right[i] * n).pvalue > P_CUT / len(words)
        if chisquare(obs, wrong[i] * n).pvalue < 1e-12:
            rejected_wrong += 1
    # the other self-exclusion convention is detected (power check, X2)
    assert rejected_wrong >= len(words) // 2


def test_sweep_tokens_pairwise_independent():
    """Within one SWEEP every token draws against frozen counts, so two
    tokens' new topics are independent (in SEQUENTIAL mode they are not)."""
    V, K = 3, 3
    doc_ptr, words = _corpus(MICRO8)
    z0 = np.array([1, 2, 0, 0, 2, 1, 0, 1], np.uint16)
    n = 60_000
    zs = O.run_chains(doc_ptr, words, V, K, ALPHA, BETA, 77, n, 1, "sweep", 0, z0)
    zq = O.run_chains(doc_ptr, words, V, K, ALPHA, BETA, 77, n, 1, "sequential", 0, z0)

    def indep_p(z, a, b):
        tab = np.zeros((K, K)); np.add.at(tab, (z[:, a], z[:, b]), 1)
        exp = np.outer(tab.sum(1), tab.sum(0)) / n
        stat = ((tab - exp) ** 2 / np.where(exp > 0, exp, 1)).sum()
        return chi2.sf(stat, (K - 1) ** 2)

    # tokens 1 and 2 share doc 0 (and token 2/3 share word 1)
    assert indep_p(zs, 1, 2) > P_CUT
    assert indep_p(zs, 2, 4) > P_CUT
    assert indep_p(zq, 1, 2) < 1e-6          # sequential scan couples them


# --------------------------------------------------------------------------
# exact laws on K^N states
# --------------------------------------------------------------------------

def _states(N, K):
    return np.array(list(itertools.product(range(K), repeat=N)), np.int64)[:, ::-1]


def _state_index(z, K):
    return (z.astype(np.int64) * (K ** np.arange(z.shape[1]))).sum(1)


def _log_joint(doc_ptr, words, z, V, K):
    """Collapsed joint log p(w, z | α, β) (Dirichlet-multinomial closed form)."""
    nwk, ndk, nk, d = _counts(doc_ptr, words, z, V, K)
    L = np.diff(doc_ptr)
    return ((gammaln(ndk + ALPHA).sum() - gammaln(L + K * ALPHA).sum())
            + (gammaln(nwk + BETA).sum() - gammaln(nk + V * BETA).sum()))


def _posterior(doc_ptr, words, V, K):
    S = _states(len(words), K)
    lj = np.array([_log_joint(doc_ptr, words, s, V, K) for s in S])
    p = np.exp(lj - lj.max())
    return p / p.sum()


def _sweep_transition(doc_ptr, words, V, K):
    S = _states(len(words), K)
    Tm = np.empty((len(S), len(S)))
    for a, s in enumerate(S):
        P = _eq1(doc_ptr, words, s, V, K, 0)
        Tm[a] = np.prod(P[np.arange(len(words))[None, :], S], axis=1)
    return Tm


def _stationary(Tm):
    w, v = np.linalg.eig(Tm.T)
    i = np.argmin(np.abs(w - 1))
    pi = np.real(v[:, i]); pi /= pi.sum()
    lam2 = np.sort(np.abs(w))[-2]
    return pi, lam2


@pytest.mark.parametrize("docs,K,n", [(MICRO8, 2, 60_000), (MICRO5, 3, 60_000)])
def test_sequential_chain_hits_exact_posterior(docs, K, n):
    V = 3
    doc_ptr, words = _corpus(docs)
    post = _posterior(doc_ptr, words, V, K)
    zf = O.run_chains(doc_ptr, words, V, K, ALPHA, BETA, seed0=5000, n_chains=n,
                      n_sweeps=100, mode="sequential")
    obs = np.bincount(_state_index(zf, K), minlength=K ** len(words))
    assert _pooled_chisq(obs, post * n) > P_CUT


@pytest.mark.parametrize("docs,K,n", [(MICRO8, 2, 40_000), (MICRO5, 3, 60_000)])
def test_sweep_chain_hits_its_stationary_law(docs, K, n):
    V = 3
    doc_ptr, words = _corpus(docs)
    Tm = _sweep_transition(doc_ptr, words, V, K)
    assert np.allclose(Tm.sum(1), 1.0)
    pi, lam2 = _stationary(Tm)
    burn = int(np.ceil(np.log(1e-6) / np.log(lam2)))
    assert burn < 1000
    zf = O.run_chains(doc_ptr, words, V, K, ALPHA, BETA, seed0=9000, n_chains=n,
                      n_sweeps=burn, mode="sweep")
    obs = np.bincount(_state_index(zf, K), minlength=K ** len(words))
    assert _pooled_chisq(obs, pi * n) > P_CUT
    # ... and the synchronous chain's law is not the posterior (X2/X3):
    post = _posterior(doc_ptr, words, V, K)
    assert 0.5 * np.abs(pi - post).sum() > 0.05
    assert _pooled_chisq(obs, post * n) < 1e-9
