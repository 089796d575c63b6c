"""Shared helpers of the GPU parity tests: run the CUDA path (through the C
ABI) and the oracle on the same seeded inputs and compare them by the
north_star rules (BASELINE.json):
  * counts bit-exact (integers);
  * per-token z identical except where the oracle's uniform lies within 1e-6
    (relative) of a CDF boundary, and such tokens < 1e-4 of all tokens;
  * LL/token within 1e-3 relative.
"""
import numpy as np

from oracle import oracle as O

MARGIN_EXCUSE = 1e-6       # north_star: "within 1e-6 relative of a CDF boundary"
MAX_EXCUSED_FRAC = 1e-4    # north_star: "fewer than 1e-4 of all tokens"
LL_RTOL = 1e-3             # north_star: LL/token "within 1e-3 relative"


def gpu_model(D, V, K, alpha, beta, doc_ptr, words, seed, **opts):
    import paper_conf_hpdc_xie0lt19_b200 as L
    m = L.LDA(D, V, K, alpha, beta, **opts)
    m.load(doc_ptr, words, seed)
    return m


def compare_z(z_gpu, z_orc, margins):
    """Returns (#mismatches, #unexcused)."""
    bad = np.nonzero(z_gpu != z_orc)[0]
    unexcused = int((margins[bad] >= MARGIN_EXCUSE).sum()) if len(bad) else 0
    return len(bad), unexcused


def check_counts_equal(g, o):
    """GPU model g vs OracleLDA o: n_wk, n_k, dense n_dk bit-exact."""
    assert np.array_equal(g.nwk(), o.nwk()), "n_wk differs"
    assert np.array_equal(g.nk(), o.n_k), "n_k differs"
    assert np.array_equal(g.ndk_dense(), o.ndk()), "n_dk differs"


def check_invariants_gpu(g, doc_ptr, words):
    """Count invariants of the GPU state alone (any size): Eq. 5 (L1011-1015),
    Σ_k n_wk = #tokens of w, n_k = Σ_w n_wk, θ rows ascending with positive
    counts and nnz_d <= min(L_d, K)."""
    V, K = g.V, g.K
    nwk = g.nwk()
    nk = g.nk()
    wc = np.bincount(words, minlength=V)
    assert np.array_equal(nwk.sum(1, dtype=np.int64), wc)
    assert np.array_equal(nwk.sum(0, dtype=np.int64), nk.astype(np.int64))
    assert (nwk >= 0).all()
    ptr, top, cnt = g.theta_csr()
    Ld = np.diff(doc_ptr)
    nnz = np.diff(ptr)
    assert (cnt > 0).all()
    assert (nnz <= np.minimum(Ld, K)).all()
    rows = np.repeat(np.arange(len(Ld)), nnz)
    assert np.array_equal(np.bincount(rows, weights=cnt, minlength=len(Ld)).astype(np.int64), Ld)
    # ascending topics within each row
    t = top.astype(np.int64)
    same_row = rows[1:] == rows[:-1]
    assert (t[1:][same_row] > t[:-1][same_row]).all()
    return nnz


def lockstep(g, o, sweeps, exclude_self=0, teacher_force=True):
    """Advance GPU and oracle together; per sweep compare z (with the excuse
    rule) and, when z agree, the counts bit-exactly.  With teacher_force the
    GPU is reset to the oracle's state after any (excused) mismatch so one
    boundary flip does not cascade.  Returns total (mismatches, unexcused)."""
    tot_bad = tot_unexc = 0
    for _ in range(sweeps):
        margins = o.iterate(1, exclude_self=exclude_self, margins=True)
        g.iterate(1)
        zg = g.z()
        bad, unexc = compare_z(zg, o.z, margins)
        tot_bad += bad
        tot_unexc += unexc
        if bad and teacher_force:
            g.set_z(o.z)
        if bad == 0 or teacher_force:
            check_counts_equal(g, o)
    return tot_bad, tot_unexc


def oracle_for(D, V, K, alpha, beta, doc_ptr, words, seed):
    return O.OracleLDA(D, V, K, alpha, beta).load(doc_ptr, words, seed)
