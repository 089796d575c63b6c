"""B200-native LDA collapsed-Gibbs sweep (the CuLDA_CGS hot path).

Thin ctypes binding of the C ABI in ``include/lda.h`` (argument marshalling
only; every step of the sweep runs in the library's CUDA kernels).  The
functions keep the ABI's names; :class:`LDA` strings them together.

The library ``liblda.so`` is built in-tree by ``_build.build()``
(``__graft_entry__.build()``).  There is no fallback: if the library is
missing or the GPU is absent the calls raise ``LDAError``.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("LDA_LIBRARY") or os.path.join(_PKG, "liblda.so")

LDA_OK, LDA_EINVAL, LDA_ERANGE, LDA_ENOMEM, LDA_ECUDA, LDA_ENCCL, LDA_ESTATE = 0, -1, -2, -3, -4, -5, -6
STATUS = {0: "LDA_OK", -1: "LDA_EINVAL", -2: "LDA_ERANGE", -3: "LDA_ENOMEM", -4: "LDA_ECUDA",
          -5: "LDA_ENCCL", -6: "LDA_ESTATE"}

# every symbol include/lda.h declares
ABI_SYMBOLS = ("lda_create", "lda_set_option", "lda_init_dist", "lda_nccl_unique_id", "lda_peer_group_create",
               "lda_init_peer", "lda_peer_group_destroy", "lda_partition_docs",
               "lda_canonical_bases", "lda_layout_selfcheck", "lda_debug_radix_sort", "lda_debug_nccl_selftest",
               "lda_load_corpus", "lda_iterate", "lda_loglik", "lda_get_counts", "lda_get_stats",
               "lda_get_sweep_log", "lda_get_loglik_log", "lda_get_stream", "lda_set_z", "lda_destroy",
               "lda_last_error", "lda_version")


class LDAError(RuntimeError):
    def __init__(self, code, msg=""):
        self.code = code
        super().__init__(f"{STATUS.get(code, code)}: {msg}")


class lda_stats(ctypes.Structure):
    _fields_ = [("sweeps_done", ctypes.c_int64), ("local_tokens", ctypes.c_int64),
                ("local_docs", ctypes.c_int64), ("global_tokens", ctypes.c_int64),
                ("last_n", ctypes.c_int32), ("world", ctypes.c_int32),
                ("ms_total", ctypes.c_double), ("ms_sample", ctypes.c_double),
                ("ms_recount", ctypes.c_double), ("ms_theta", ctypes.c_double),
                ("ms_allreduce", ctypes.c_double), ("ms_last_sweep", ctypes.c_double),
                ("ms_last_sample", ctypes.c_double), ("sum_nnz_tok", ctypes.c_int64),
                ("sum_nnz_doc", ctypes.c_int64), ("n_launches", ctypes.c_int64),
                ("n_sample_chunks", ctypes.c_int64), ("n_exact_redraws", ctypes.c_int64),
                ("ms_table", ctypes.c_double), ("ms_allreduce_exposed", ctypes.c_double),
                ("tile_tokens", ctypes.c_int64), ("n_tiles", ctypes.c_int32), ("sampler", ctypes.c_int32),
                ("bytes_alg", ctypes.c_double), ("bytes_sample", ctypes.c_double),
                ("n_stream_chunks", ctypes.c_int64), ("n_sparse_words", ctypes.c_int64)]

    def as_dict(self):
        return {f: getattr(self, f) for f, _ in self._fields_}


_lib = None
_vp = ctypes.c_void_p
_i64, _i32, _u64, _f64 = ctypes.c_int64, ctypes.c_int32, ctypes.c_uint64, ctypes.c_double


def lib():
    """Load liblda.so (raises if it has not been built)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise LDAError(LDA_ECUDA, f"{LIB_PATH} not built; run __graft_entry__.build()")
        L = ctypes.CDLL(LIB_PATH)
        sig = {
            "lda_create": ([_i64, _i32, _i32, _f64, _f64, ctypes.POINTER(_vp)], ctypes.c_int),
            "lda_set_option": ([_vp, ctypes.c_char_p, _i64], ctypes.c_int),
            "lda_init_dist": ([_vp, _i32, _i32, _vp], ctypes.c_int),
            "lda_nccl_unique_id": ([_vp], ctypes.c_int),
            "lda_peer_group_create": ([_i32, ctypes.POINTER(_vp)], ctypes.c_int),
            "lda_init_peer": ([_vp, _vp, _i32], ctypes.c_int),
            "lda_peer_group_destroy": ([_vp], None),
            "lda_get_loglik_log": ([_vp, _i32, _vp, _vp, ctypes.POINTER(_i32)], ctypes.c_int),
            "lda_partition_docs": ([_i64, _vp, _i32, _vp], ctypes.c_int),
            "lda_canonical_bases": ([_i32, _i32, _i32, _vp, _vp, ctypes.POINTER(_i64)], ctypes.c_int),
            "lda_layout_selfcheck": ([_i64, _i32, _i32, _vp, _vp, _i32, _i64, _i64, _i64, _vp, ctypes.c_char_p,
                                      _i32], ctypes.c_int),
            "lda_load_corpus": ([_vp, _i64, _i64, _vp, _vp, _u64], ctypes.c_int),
            "lda_debug_radix_sort": ([_vp, _vp, _i64, _i32, _vp, _vp], ctypes.c_int),
            "lda_debug_nccl_selftest": ([_i32, ctypes.c_char_p, _i32], ctypes.c_int),
            "lda_iterate": ([_vp, _i32], ctypes.c_int),
            "lda_loglik": ([_vp, ctypes.POINTER(_f64)], ctypes.c_int),
            "lda_get_counts": ([_vp, _vp, _vp, _vp, _vp, _vp, _i64, _vp, _vp], ctypes.c_int),
            "lda_get_stats": ([_vp, ctypes.POINTER(lda_stats)], ctypes.c_int),
            "lda_get_sweep_log": ([_vp, _i32, _vp, _vp, _vp, _vp, _vp, _vp, _vp, _vp], ctypes.c_int),
            "lda_get_stream": ([_vp, ctypes.POINTER(_vp)], ctypes.c_int),
            "lda_set_z": ([_vp, _vp], ctypes.c_int),
            "lda_destroy": ([_vp], None),
            "lda_last_error": ([_vp], ctypes.c_char_p),
            "lda_version": ([], ctypes.c_char_p),
        }
        for name, (args, res) in sig.items():
            f = getattr(L, name)
            f.argtypes = args
            f.restype = res
        _lib = L
    return _lib


def _p(a):
    return None if a is None else a.ctypes.data_as(_vp)


def _check(rc, ctx=None):
    if rc != LDA_OK:
        msg = lib().lda_last_error(ctx).decode() if ctx else ""
        raise LDAError(rc, msg)


# ---------------------------------------------------------------------------
# same-name wrappers of the C ABI
# ---------------------------------------------------------------------------

def lda_version() -> str:
    return lib().lda_version().decode()


def lda_create(D, V, K, alpha, beta):
    h = _vp()
    _check(lib().lda_create(int(D), int(V), int(K), float(alpha), float(beta), ctypes.byref(h)))
    return h


def lda_set_option(ctx, key, value):
    _check(lib().lda_set_option(ctx, key.encode(), int(value)), ctx)


def lda_nccl_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(lib().lda_nccl_unique_id(buf))
    return buf.raw


def lda_init_dist(ctx, rank, world, unique_id: bytes | None):
    buf = ctypes.create_string_buffer(unique_id, 128) if unique_id is not None else None
    _check(lib().lda_init_dist(ctx, int(rank), int(world), buf), ctx)


def lda_partition_docs(doc_ptr, world):
    doc_ptr = np.ascontiguousarray(doc_ptr, np.int64)
    out = np.empty(int(world) + 1, np.int64)
    _check(lib().lda_partition_docs(len(doc_ptr) - 1, _p(doc_ptr), int(world), _p(out)))
    return out


def lda_layout_selfcheck(doc_ptr, words, V, K, sampler=2, tile_tokens=0, chunk_tokens=4096, tail_per_tile=64):
    """Host-only check of the token layout (include/lda.h); returns
    {tiles, items, tail_words, runs} or raises LDAError with the failed invariant."""
    doc_ptr = np.ascontiguousarray(doc_ptr, np.int64)
    words = np.ascontiguousarray(words, np.int32)
    st = np.zeros(4, np.int64)
    buf = ctypes.create_string_buffer(256)
    r = lib().lda_layout_selfcheck(len(doc_ptr) - 1, int(V), int(K), _p(doc_ptr), _p(words), int(sampler),
                                   int(tile_tokens), int(chunk_tokens), int(tail_per_tile), _p(st), buf, 256)
    if r != 0:
        raise LDAError(r, f"lda_layout_selfcheck: {buf.value.decode()}")
    return dict(zip(("tiles", "items", "tail_words", "runs"), st.tolist()))


def lda_debug_radix_sort(keys, vals, bits):
    """The library's stable device radix sort (diagnostic): returns (keys, vals) sorted by the low `bits` key bits."""
    k = np.ascontiguousarray(keys, np.uint32)
    v = np.ascontiguousarray(vals, np.uint32)
    if k.shape != v.shape:
        raise LDAError(LDA_EINVAL, "keys and vals differ in length")
    ok, ov = np.empty_like(k), np.empty_like(v)
    _check(lib().lda_debug_radix_sort(_p(k), _p(v), len(k), int(bits), _p(ok), _p(ov)))
    return ok, ov


def lda_debug_nccl_selftest(device=0) -> str:
    """The NCCL backend end to end with one rank (diagnostic); returns its message."""
    buf = ctypes.create_string_buffer(512)
    r = lib().lda_debug_nccl_selftest(int(device), buf, 512)
    if r != LDA_OK:
        raise LDAError(r, buf.value.decode())
    return buf.value.decode()


def lda_canonical_bases(word_counts, rank):
    """word_counts: (world, V) int64 per-rank word histograms -> (cbase[V], T)."""
    wc = np.ascontiguousarray(word_counts, np.int64)
    world, V = wc.shape
    out = np.empty(V, np.int64)
    tot = _i64()
    _check(lib().lda_canonical_bases(V, world, int(rank), _p(wc), _p(out), ctypes.byref(tot)))
    return out, tot.value


def lda_load_corpus(ctx, doc_begin, doc_end, doc_ptr, words, seed):
    doc_ptr = np.ascontiguousarray(doc_ptr, np.int64)
    words = np.ascontiguousarray(words, np.int32)
    # the C side reads doc_ptr[0 .. doc_end-doc_begin] and words[0 .. doc_ptr[-1])
    if doc_ptr.ndim != 1 or len(doc_ptr) != int(doc_end) - int(doc_begin) + 1:
        raise LDAError(LDA_EINVAL, "len(doc_ptr) must be doc_end - doc_begin + 1")
    if len(doc_ptr) and (doc_ptr[-1] < 0 or len(words) < int(doc_ptr[-1])):
        raise LDAError(LDA_EINVAL, "len(words) must be >= doc_ptr[-1]")
    _check(lib().lda_load_corpus(ctx, int(doc_begin), int(doc_end), _p(doc_ptr), _p(words),
                                 int(seed) & 0xFFFFFFFFFFFFFFFF), ctx)


def lda_iterate(ctx, n):
    _check(lib().lda_iterate(ctx, int(n)), ctx)


def lda_loglik(ctx) -> float:
    v = _f64()
    _check(lib().lda_loglik(ctx, ctypes.byref(v)), ctx)
    return v.value


def _out(a, dtype, n, name):
    if a is None:
        return
    if a.dtype != dtype or not a.flags.c_contiguous or a.size < n:
        raise LDAError(LDA_EINVAL, f"{name} must be a C-contiguous {np.dtype(dtype).name} array of >= {n} entries")


def lda_get_counts(ctx, n_wk=None, n_k=None, ndk_ptr=None, ndk_topic=None, ndk_count=None, z=None,
                   want_nnz=False, shape=None):
    """Fills the given (preallocated, C-contiguous) numpy arrays; returns nnz.
    shape = (V, K, D_g, T_g) enables the size checks (LDA does this)."""
    if shape is not None:
        V, K, Dg, Tg = shape
        _out(n_wk, np.int32, V * K, "n_wk")
        _out(n_k, np.int32, K, "n_k")
        _out(ndk_ptr, np.int64, Dg + 1, "ndk_ptr")
        _out(z, np.uint16, Tg, "z")
    _out(ndk_topic, np.uint16, 0, "ndk_topic")
    _out(ndk_count, np.int32, 0, "ndk_count")
    nnz = _i64()
    cap = 0 if ndk_topic is None else len(ndk_topic)
    if ndk_count is not None:
        cap = len(ndk_count) if ndk_topic is None else min(cap, len(ndk_count))
    # the θ rows are read back (and nnz counted) only when a θ array is requested
    want = want_nnz or ndk_ptr is not None or ndk_topic is not None or ndk_count is not None
    _check(lib().lda_get_counts(ctx, _p(n_wk), _p(n_k), _p(ndk_ptr), _p(ndk_topic), _p(ndk_count), cap,
                                ctypes.byref(nnz) if want else None, _p(z)), ctx)
    return nnz.value if want else None


def lda_get_stats(ctx) -> dict:
    s = lda_stats()
    _check(lib().lda_get_stats(ctx, ctypes.byref(s)), ctx)
    return s.as_dict()


def lda_get_sweep_log(ctx) -> dict:
    n = _i32()
    _check(lib().lda_get_sweep_log(ctx, 0, None, None, None, None, None, None, None, ctypes.byref(n)), ctx)
    m = n.value
    arr = {k: np.zeros(m, np.float64) for k in ("ms_sweep", "ms_sample", "ms_recount", "ms_theta", "ms_allreduce")}
    nnz = np.zeros(m, np.int64)
    nnzd = np.zeros(m, np.int64)
    _check(lib().lda_get_sweep_log(ctx, m, _p(arr["ms_sweep"]), _p(arr["ms_sample"]), _p(arr["ms_recount"]),
                                   _p(arr["ms_theta"]), _p(arr["ms_allreduce"]), _p(nnz), _p(nnzd),
                                   ctypes.byref(n)), ctx)
    arr["sum_nnz_tok"] = nnz
    arr["sum_nnz_doc"] = nnzd
    return arr


def lda_get_loglik_log(ctx) -> dict:
    n = _i32()
    _check(lib().lda_get_loglik_log(ctx, 0, None, None, ctypes.byref(n)), ctx)
    sw = np.zeros(n.value, np.int64)
    ll = np.zeros(n.value, np.float64)
    _check(lib().lda_get_loglik_log(ctx, n.value, _p(sw), _p(ll), ctypes.byref(n)), ctx)
    return {"sweep": sw, "ll_per_token": ll}


def lda_peer_group_create(world):
    h = _vp()
    _check(lib().lda_peer_group_create(int(world), ctypes.byref(h)))
    return h


def lda_init_peer(ctx, group, rank):
    _check(lib().lda_init_peer(ctx, group, int(rank)), ctx)


def lda_peer_group_destroy(group):
    if group:
        lib().lda_peer_group_destroy(group)


class PeerGroup:
    """In-process group of `world` ranks (include/lda.h lda_peer_group_*):
    each rank's LDA is driven by its own thread; the n_wk/n_k exchange reads
    the peers' device buffers directly."""

    def __init__(self, world):
        self.world = int(world)
        self.h = lda_peer_group_create(self.world)

    def close(self):
        if self.h:
            lda_peer_group_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def lda_get_stream(ctx) -> int:
    s = _vp()
    _check(lib().lda_get_stream(ctx, ctypes.byref(s)), ctx)
    return int(s.value or 0)


def lda_set_z(ctx, z, T=None):
    z = np.ascontiguousarray(z, np.uint16)
    if T is not None and z.shape != (int(T),):
        raise LDAError(LDA_EINVAL, f"z must hold exactly T = {T} topics")
    _check(lib().lda_set_z(ctx, _p(z)), ctx)


def lda_destroy(ctx):
    if ctx:
        lib().lda_destroy(ctx)


def lda_last_error(ctx) -> str:
    return lib().lda_last_error(ctx).decode()


# ---------------------------------------------------------------------------
# convenience object
# ---------------------------------------------------------------------------

class LDA:
    """One rank's sampler: create -> [options] -> [dist] -> load -> iterate."""

    def __init__(self, D, V, K, alpha=None, beta=0.01, **options):
        self.D, self.V, self.K = int(D), int(V), int(K)
        self.alpha = 50.0 / K if alpha is None else float(alpha)
        self.beta = float(beta)
        self.ctx = lda_create(self.D, self.V, self.K, self.alpha, self.beta)
        for k, v in options.items():
            lda_set_option(self.ctx, k, v)
        self.doc_begin, self.doc_end = 0, self.D
        self.T = 0

    def init_dist(self, rank, world, unique_id):
        lda_init_dist(self.ctx, rank, world, unique_id)

    def init_peer(self, group, rank):
        lda_init_peer(self.ctx, group.h if isinstance(group, PeerGroup) else group, rank)

    def load(self, doc_ptr, words, seed, doc_begin=0, doc_end=None):
        self.doc_begin = int(doc_begin)
        self.doc_end = self.D if doc_end is None else int(doc_end)
        self.doc_ptr = np.ascontiguousarray(doc_ptr, np.int64)
        self.T = int(self.doc_ptr[-1])
        lda_load_corpus(self.ctx, self.doc_begin, self.doc_end, self.doc_ptr, words, seed)
        return self

    def iterate(self, n=1):
        lda_iterate(self.ctx, n)

    def loglik(self):
        return lda_loglik(self.ctx)

    def z(self, out=None):
        """z in document order; `out` (uint16[T], e.g. a pinned buffer) is
        filled in place when given."""
        if out is None:
            out = np.empty(self.T, np.uint16)
        elif out.dtype != np.uint16 or out.shape != (self.T,) or not out.flags.c_contiguous:
            raise ValueError("out must be a contiguous uint16 array of T entries")
        lda_get_counts(self.ctx, z=out, shape=self._shape())
        return out

    def _shape(self):
        return (self.V, self.K, self.doc_end - self.doc_begin, self.T)

    def set_z(self, z):
        lda_set_z(self.ctx, z, T=self.T)

    def nwk(self):
        a = np.empty(self.V * self.K, np.int32)
        lda_get_counts(self.ctx, n_wk=a, shape=self._shape())
        return a.reshape(self.V, self.K)

    def nk(self):
        a = np.empty(self.K, np.int32)
        lda_get_counts(self.ctx, n_k=a, shape=self._shape())
        return a

    def theta_csr(self):
        nnz = lda_get_counts(self.ctx, want_nnz=True)
        Dg = self.doc_end - self.doc_begin
        ptr = np.empty(Dg + 1, np.int64)
        top = np.empty(nnz, np.uint16)
        cnt = np.empty(nnz, np.int32)
        lda_get_counts(self.ctx, ndk_ptr=ptr, ndk_topic=top, ndk_count=cnt, shape=self._shape())
        return ptr, top, cnt

    def ndk_dense(self):
        ptr, top, cnt = self.theta_csr()
        Dg = len(ptr) - 1
        out = np.zeros((Dg, self.K), np.int32)
        rows = np.repeat(np.arange(Dg), np.diff(ptr))
        out[rows, top.astype(np.int64)] = cnt
        return out

    def stats(self):
        return lda_get_stats(self.ctx)

    def sweep_log(self):
        return lda_get_sweep_log(self.ctx)

    def loglik_log(self):
        return lda_get_loglik_log(self.ctx)

    def stream(self):
        return lda_get_stream(self.ctx)

    def close(self):
        if self.ctx:
            lda_destroy(self.ctx)
            self.ctx = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()
