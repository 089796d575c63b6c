"""ctypes wrapper of oracle/lda_oracle.c — TEST INFRASTRUCTURE ONLY.

Only tests/, ``__graft_entry__.smoke()`` and bench.py's ``cpu_baseline`` /
``--impl reference`` legs may import this module.  It is argument
marshalling only: every step of the oracle's arithmetic is in
lda_oracle.c (see its header for the paper citations and pins).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "lda_oracle.c")
_LIB = os.path.join(_HERE, "liblda_oracle.so")

_i64p = np.ctypeslib.ndpointer(np.int64, flags="C_CONTIGUOUS")
_i32p = np.ctypeslib.ndpointer(np.int32, flags="C_CONTIGUOUS")
_u16p = np.ctypeslib.ndpointer(np.uint16, flags="C_CONTIGUOUS")
_u32p = np.ctypeslib.ndpointer(np.uint32, flags="C_CONTIGUOUS")
_f64p = np.ctypeslib.ndpointer(np.float64, flags="C_CONTIGUOUS")


def build_oracle(force: bool = False) -> str:
    """Compile the C oracle (plain gcc, IEEE fp64, no FMA contraction)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        cmd = ["gcc", "-std=c11", "-O2", "-fPIC", "-shared", "-ffp-contract=off",
               "-fno-fast-math", "-fopenmp", _SRC, "-o", _LIB + ".tmp", "-lm"]
        subprocess.check_call(cmd)
        os.replace(_LIB + ".tmp", _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = ctypes.CDLL(build_oracle())
        c = ctypes
        L.orc_philox4x32_10.argtypes = [_u32p, _u32p, _u32p]
        L.orc_philox4x32_10.restype = None
        L.orc_token_x0.argtypes = [c.c_uint64, c.c_uint64, c.c_uint32]
        L.orc_token_x0.restype = c.c_uint32
        L.orc_canonical_order.argtypes = [c.c_int64, c.c_int32, _i64p, _i32p, _i64p]
        L.orc_canonical_order.restype = None
        L.orc_canonical_index_of.argtypes = [c.c_int64, c.c_int32, _i64p, _i32p,
                                             c.c_int64, _i64p, _i64p]
        L.orc_canonical_index_of.restype = None
        L.orc_init_topic.argtypes = [c.c_uint64, c.c_uint64, c.c_int32]
        L.orc_init_topic.restype = c.c_uint16
        L.orc_init.argtypes = [c.c_int64, _i64p, c.c_int32, c.c_uint64, _u16p]
        L.orc_init.restype = None
        L.orc_init_range_hist.argtypes = [c.c_uint64, c.c_int64, c.c_int64, c.c_int32, _i32p]
        L.orc_init_range_hist.restype = None
        L.orc_counts.argtypes = [c.c_int64, c.c_int32, c.c_int32, _i64p, _i32p, _u16p,
                                 _i32p, _i32p, c.c_void_p]
        L.orc_counts.restype = None
        L.orc_check_invariants.argtypes = [c.c_int64, c.c_int32, c.c_int32, _i64p, _i32p,
                                           _i32p, _i32p, c.c_void_p]
        L.orc_check_invariants.restype = c.c_int
        L.orc_search.argtypes = [_f64p, c.c_int64, c.c_double]
        L.orc_search.restype = c.c_int64
        L.orc_draw.argtypes = [c.c_int32, c.c_int32, c.c_double, c.c_double, _i32p, _i32p,
                               _i32p, c.c_int, c.c_int32, c.c_uint32,
                               c.POINTER(c.c_double)]
        L.orc_draw.restype = c.c_int32
        L.orc_sweep.argtypes = [c.c_int64, c.c_int32, c.c_int32, c.c_double, c.c_double,
                                _i64p, _i32p, _i64p, c.c_uint64, c.c_uint32, c.c_int,
                                _u16p, _i32p, _i32p, _i32p, c.c_void_p]
        L.orc_sweep.restype = None
        L.orc_draw_docs.argtypes = [c.c_int64, c.c_int64, c.c_int32, c.c_int32, c.c_double,
                                    c.c_double, _i64p, _i32p, _i64p, c.c_uint64, c.c_uint32,
                                    c.c_int, _u16p, _i32p, _i32p, _i32p, _u16p, c.c_void_p]
        L.orc_draw_docs.restype = None
        L.orc_sweep_omp.argtypes = L.orc_sweep.argtypes
        L.orc_sweep_omp.restype = None
        L.orc_omp_threads.argtypes = []
        L.orc_omp_threads.restype = c.c_int
        L.orc_sweep_sequential.argtypes = [c.c_int64, c.c_int32, c.c_int32, c.c_double,
                                           c.c_double, _i64p, _i32p, _i64p, c.c_uint64,
                                           c.c_uint32, _u16p, _i32p, _i32p, _i32p]
        L.orc_sweep_sequential.restype = None
        L.orc_loglik.argtypes = [c.c_int64, c.c_int32, c.c_int32, c.c_double, c.c_double,
                                 _i64p, _i32p, _i32p, _i32p]
        L.orc_loglik.restype = c.c_double
        L.orc_run_chains.argtypes = [c.c_int64, c.c_int32, c.c_int32, c.c_double,
                                     c.c_double, _i64p, _i32p, _i64p, c.c_uint64,
                                     c.c_int64, c.c_int32, c.c_int, c.c_int, c.c_void_p,
                                     _u16p]
        L.orc_run_chains.restype = None
        _lib = L
    return _lib


def _vp(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


# ---------------------------------------------------------------------------
# thin function wrappers
# ---------------------------------------------------------------------------

def philox4x32_10(ctr, key):
    out = np.zeros(4, np.uint32)
    lib().orc_philox4x32_10(np.ascontiguousarray(ctr, np.uint32),
                            np.ascontiguousarray(key, np.uint32), out)
    return out


def token_x0(seed: int, c: int, t: int) -> int:
    return int(lib().orc_token_x0(seed, c, t))


def canonical_order(doc_ptr, words, V):
    doc_ptr = np.ascontiguousarray(doc_ptr, np.int64)
    words = np.ascontiguousarray(words, np.int32)
    canon = np.empty(len(words), np.int64)
    lib().orc_canonical_order(len(doc_ptr) - 1, V, doc_ptr, words, canon)
    return canon


def canonical_index_of(doc_ptr, words, V, query):
    doc_ptr = np.ascontiguousarray(doc_ptr, np.int64)
    words = np.ascontiguousarray(words, np.int32)
    q = np.asarray(query, np.int64)
    order = np.argsort(q, kind="stable")
    qs = np.ascontiguousarray(q[order])
    out_s = np.empty(len(qs), np.int64)
    lib().orc_canonical_index_of(len(doc_ptr) - 1, V, doc_ptr, words, len(qs), qs, out_s)
    out = np.empty_like(out_s)
    out[order] = out_s
    return out


def init_topic(seed, c, K):
    return int(lib().orc_init_topic(seed, c, K))


def init_range_hist(seed, c_begin, n, K, hist=None):
    if hist is None:
        hist = np.zeros(K, np.int32)
    lib().orc_init_range_hist(seed, c_begin, n, K, hist)
    return hist


def search(prefix, x):
    p = np.ascontiguousarray(prefix, np.float64)
    return int(lib().orc_search(p, len(p), float(x)))


def draw(K, V, alpha, beta, nwk_row, n_k, ndk_row, x0, exclude_self=0, z_old=-1):
    m = ctypes.c_double()
    z = lib().orc_draw(K, V, alpha, beta, np.ascontiguousarray(nwk_row, np.int32),
                       np.ascontiguousarray(n_k, np.int32),
                       np.ascontiguousarray(ndk_row, np.int32), exclude_self, z_old,
                       x0, ctypes.byref(m))
    return int(z), m.value


def draw_docs(d_begin, d_end, doc_ptr, words, canon, V, K, alpha, beta, seed, t, z, n_wk, n_k,
              n_dk, exclude_self=0, margins=False):
    """New topics of the tokens of documents [d_begin, d_end) against the given
    global counts (input order; other entries of the result are 0).  canon[i]
    is token i's global canonical index, n_dk the dense rows of these
    documents.  With margins=True also returns each token's margin."""
    z = np.ascontiguousarray(z, np.uint16)
    out = np.zeros_like(z)
    m = np.full(len(z), np.inf) if margins else None
    lib().orc_draw_docs(d_begin, d_end, V, K, alpha, beta, np.ascontiguousarray(doc_ptr, np.int64),
                        np.ascontiguousarray(words, np.int32), np.ascontiguousarray(canon, np.int64),
                        seed, t, exclude_self, z, np.ascontiguousarray(n_wk, np.int32).reshape(-1),
                        np.ascontiguousarray(n_k, np.int32), np.ascontiguousarray(n_dk, np.int32).reshape(-1),
                        out, _vp(m))
    return (out, m) if margins else out


def omp_threads() -> int:
    return int(lib().orc_omp_threads())


def loglik(doc_ptr, V, K, alpha, beta, n_wk, n_k, n_dk):
    doc_ptr = np.ascontiguousarray(doc_ptr, np.int64)
    return float(lib().orc_loglik(len(doc_ptr) - 1, V, K, alpha, beta, doc_ptr,
                                  np.ascontiguousarray(n_wk, np.int32).reshape(-1),
                                  np.ascontiguousarray(n_k, np.int32),
                                  np.ascontiguousarray(n_dk, np.int32).reshape(-1)))


def run_chains(doc_ptr, words, V, K, alpha, beta, seed0, n_chains, n_sweeps,
               mode="sweep", exclude_self=0, z_start=None):
    doc_ptr = np.ascontiguousarray(doc_ptr, np.int64)
    words = np.ascontiguousarray(words, np.int32)
    canon = canonical_order(doc_ptr, words, V)
    T = len(words)
    out = np.empty(n_chains * T, np.uint16)
    zs = None if z_start is None else np.ascontiguousarray(z_start, np.uint16)
    lib().orc_run_chains(len(doc_ptr) - 1, V, K, alpha, beta, doc_ptr, words, canon,
                         seed0, n_chains, n_sweeps, 0 if mode == "sweep" else 1,
                         exclude_self, _vp(zs), out)
    return out.reshape(n_chains, T)


class OracleLDA:
    """Whole-corpus oracle state (dense n_dk).  Mirrors the C ABI's life
    cycle: create -> load (random init, t = 0) -> iterate (t = 1, 2, ...)."""

    def __init__(self, D, V, K, alpha, beta):
        self.D, self.V, self.K = int(D), int(V), int(K)
        self.alpha, self.beta = float(alpha), float(beta)
        self.t = 0

    def load(self, doc_ptr, words, seed):
        self.doc_ptr = np.ascontiguousarray(doc_ptr, np.int64)
        self.words = np.ascontiguousarray(words, np.int32)
        assert len(self.doc_ptr) == self.D + 1
        self.T = int(self.doc_ptr[-1])
        self.seed = int(seed)
        self.canon = canonical_order(self.doc_ptr, self.words, self.V)
        self.z = np.empty(self.T, np.uint16)
        lib().orc_init(self.T, self.canon, self.K, self.seed, self.z)
        self.n_wk = np.zeros(self.V * self.K, np.int32)
        self.n_k = np.zeros(self.K, np.int32)
        self.n_dk = np.zeros(self.D * self.K, np.int32)
        self._recount()
        self.t = 0
        return self

    def _recount(self):
        lib().orc_counts(self.D, self.V, self.K, self.doc_ptr, self.words, self.z,
                         self.n_wk, self.n_k, _vp(self.n_dk))

    def set_z(self, z):
        self.z[:] = np.asarray(z, np.uint16)
        self._recount()

    def iterate(self, n=1, mode="sweep", exclude_self=0, margins=False, parallel=False):
        """mode "sweep" (the GPU semantics) or "sequential"; parallel=True runs
        the sweep's draws on all host cores (oracle-omp, bit-identical)."""
        m = np.empty(self.T, np.float64) if margins else None
        sweep = lib().orc_sweep_omp if parallel else lib().orc_sweep
        for _ in range(n):
            self.t += 1
            if mode == "sweep":
                sweep(self.D, self.V, self.K, self.alpha, self.beta,
                                self.doc_ptr, self.words, self.canon, self.seed,
                                self.t, exclude_self, self.z, self.n_wk, self.n_k,
                                self.n_dk, _vp(m))
            else:
                lib().orc_sweep_sequential(self.D, self.V, self.K, self.alpha,
                                           self.beta, self.doc_ptr, self.words,
                                           self.canon, self.seed, self.t, self.z,
                                           self.n_wk, self.n_k, self.n_dk)
        return m

    def loglik(self):
        return float(lib().orc_loglik(self.D, self.V, self.K, self.alpha, self.beta,
                                      self.doc_ptr, self.n_wk, self.n_k, self.n_dk))

    def invariants(self):
        return int(lib().orc_check_invariants(self.D, self.V, self.K, self.doc_ptr,
                                              self.words, self.n_wk, self.n_k,
                                              _vp(self.n_dk)))

    def nwk(self):
        return self.n_wk.reshape(self.V, self.K)

    def ndk(self):
        return self.n_dk.reshape(self.D, self.K)
