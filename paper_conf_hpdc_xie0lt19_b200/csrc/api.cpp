// C ABI (include/lda.h): context life cycle, corpus loading, the per-sweep
// orchestration of Alg. 1 WorkSchedule1 (M = 1, L807-835) on one GPU per
// process, and the n_wk/n_k sum-allreduce of Eq. 4 (L935-937) over NCCL.
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nccl.h>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <condition_variable>
#include <mutex>
#include <thread>
#include <cstdlib>
#include <cmath>
#include <cstring>
#include <new>
#include <string>
#include <vector>

#include "../../include/lda.h"
#include "lda_internal.h"

// f3 (Alg. 1 WorkSchedule2, L835-859; §5.1): with M > 1 a rank's
// documents are cut into M chunks whose per-token state lives in pinned host
// memory and is streamed through two device slots every sweep (the transfer
// of chunk m+1 overlaps the computation of chunk m, L925-931).
namespace lda_stream {
struct Chunk {
    lda::HostLayout H;                // token tables (tok_row, doc_map: host, page-locked), items, runs
    lda::DevState R;                  // device-resident small tables of the chunk (offsets, runs, items)
    int64_t doc_begin = 0, D = 0;     // rank-local documents [doc_begin, doc_begin + D)
    int64_t tok_begin = 0, T = 0;     // rank-local tokens
    uint16_t *hz = nullptr;           // pinned: z, word-major (the chunk's layout)
    uint32_t *hrows = nullptr;        // pinned: θ rows, rows32 * 8 words
    bool registered = false;
};
struct Slot {
    uint32_t *tok_row = nullptr, *doc_map = nullptr, *rows = nullptr;
    uint16_t *z = nullptr, *z_doc = nullptr;
    cudaEvent_t in = nullptr, done = nullptr, free_ = nullptr;
};
}  // namespace lda_stream

struct lda_ctx {
    int64_t D = 0;
    int32_t V = 0, K = 0;
    double alpha = 0, beta = 0;
    // options
    int device = 0;
    int exclude_self = 0;
    int64_t chunk_tokens = 4096;
    int64_t recount_tokens = 65536;
    int64_t tile_tokens = -1;  // auto: tiles whose θ rows fill about half the L2
    int sampler = -1;  // auto
    int64_t tail_per_tile = 48;  // measured: +1.9 % at PubMed shape over 64, neutral at NYTimes shape
    int64_t certify_slack = 1;
    int fused_recount = 0;  // segmented recount after the sampler (measured faster)
    int64_t comm_pipeline = 4;  // world > 1: word ranges whose rows are exchanged as soon as recounted (f1)
    int64_t sparse_words = 0;  // f2: words with <= this many tokens get sparse rows (-1: K/4; 0 off: measured slower)
    int threads = 0;
    // distribution: the exchange of Eq. 4 (NCCL or the in-process peer group)
    int32_t rank = 0, world = 1;
    std::unique_ptr<lda::Comm> comm;
    // state
    bool loaded = false;
    int failed = 0;
    std::string err;
    uint64_t sweeps = 0;
    int64_t T_global = 0;
    int64_t tile_tokens_used = 0;
    lda::HostLayout H;
    lda::DevState S;
    cudaStream_t stream = nullptr, comm_stream = nullptr;
    std::vector<cudaEvent_t> ev;  // 7 per sweep
    lda_stats stats{};
    std::vector<void *> allocs;
    // θ statistics: Σ_d L_d·nnz_d (= Σ_t nnz_{d(t)}) and Σ_d nnz_d of the
    // current θ, and a per-sweep log of the last lda_iterate call.
    int64_t cur_lnnz = 0, cur_nnz = 0;
    unsigned long long *d_stat_log = nullptr;
    size_t stat_log_cap = 0;
    std::vector<double> log_ms, log_ms_sample, log_ms_recount, log_ms_theta, log_ms_comm;
    std::vector<int64_t> log_nnz_tok, log_nnz_doc;
    // f1: recount work items grouped by word range; range p = items
    // [rc_begin[p], rc_begin[p+1]), rows [w_begin[p], w_begin[p+1]) of n_wk
    std::vector<int64_t> rc_begin, w_begin;
    std::vector<cudaEvent_t> range_ev;
    // f3: out-of-HBM streaming (option stream_chunks = M)
    int64_t stream_chunks = 1;
    std::vector<std::unique_ptr<lda_stream::Chunk>> chunks;
    lda_stream::Slot slot[2];
    cudaStream_t h2d_stream = nullptr, d2h_stream = nullptr;
    // option loglik_every: LL/token after every n-th sweep of lda_iterate
    int64_t loglik_every = 0;
    std::vector<int64_t> ll_sweep;
    std::vector<double> ll_value, ll_pending;
    std::vector<int64_t> gcount;  // V: global tokens per word (load)
};

// Handle of an in-process peer group (shared by its ranks' contexts).
struct lda_peer_group {
    std::shared_ptr<lda::PeerGroup> g;
};

namespace {

constexpr int32_t kMaxK = 65536;  // u16 topic ids (L1239-1243)

int fail(lda_ctx *c, int code, const std::string &msg) {
    if (c) {
        c->err = msg;
        if (code == LDA_ECUDA || code == LDA_ENCCL) c->failed = code;
    }
    return code;
}

#define CU(call)                                                                             \
    do {                                                                                     \
        cudaError_t e_ = (call);                                                             \
        if (e_ != cudaSuccess)                                                               \
            return fail(ctx, LDA_ECUDA, std::string(#call) + ": " + cudaGetErrorString(e_)); \
    } while (0)

#define KL(call)                                                                                   \
    do {                                                                                           \
        int e_ = (call);                                                                           \
        if (e_ != 0)                                                                               \
            return fail(ctx, LDA_ECUDA,                                                            \
                        std::string(#call) + ": " + cudaGetErrorString(static_cast<cudaError_t>(e_))); \
    } while (0)

// a collective of the context's communicator; failures are sticky
#define COMM(call)                                                  \
    do {                                                            \
        std::string e_;                                             \
        int r_ = ctx->comm->call;                                   \
        if (r_ != LDA_OK) {                                         \
            ctx->err = std::string(ctx->comm->name()) + ": " + e_;  \
            ctx->failed = r_ == LDA_ENCCL ? LDA_ENCCL : LDA_ECUDA;  \
            return ctx->failed;                                     \
        }                                                           \
    } while (0)

#define PRECHECK(ctx)                                   \
    do {                                                \
        if (!(ctx)) return LDA_EINVAL;                  \
        if ((ctx)->failed) return (ctx)->failed;        \
    } while (0)

template <class T>
int dalloc(lda_ctx *ctx, T **p, size_t n) {
    void *q = nullptr;
    cudaError_t e = cudaMalloc(&q, std::max<size_t>(n, 1) * sizeof(T));
    if (e != cudaSuccess) {
        cudaGetLastError();
        return fail(ctx, e == cudaErrorMemoryAllocation ? LDA_ENOMEM : LDA_ECUDA,
                    std::string("cudaMalloc(") + std::to_string(n * sizeof(T)) + " B): " + cudaGetErrorString(e));
    }
    ctx->allocs.push_back(q);
    *p = static_cast<T *>(q);
    return LDA_OK;
}

#define DA(ptr, n)                               \
    do {                                         \
        int r_ = dalloc(ctx, &(ptr), (n));       \
        if (r_ != LDA_OK) return r_;             \
    } while (0)

// f2: sparse word rows for the large-K sampler's compact tables (kernels.cu
// SparseRows): a word with at most `sparse_words` tokens in the whole corpus
// (so at most that many nonzero n_wk) gets min(count, K) entries.
int setup_sparse_rows(lda_ctx *ctx) {
    lda::DevState &S = ctx->S;
    const int32_t V = ctx->V, K = ctx->K;
    const int64_t thr = ctx->sparse_words < 0 ? K / 4 : ctx->sparse_words;
    S.sp_words = 0;
    S.sp_cap = 0;
    if (!(S.sweep_tile_cta && S.tile_cta_gnk) || (K & 3) || thr <= 0 ||
        ctx->gcount.size() != static_cast<size_t>(V))
        return LDA_OK;
    std::vector<uint32_t> off(static_cast<size_t>(V) + 1);
    uint64_t tot = 0;
    int64_t nsp = 0;
    for (int32_t w = 0; w < V; ++w) {
        off[w] = static_cast<uint32_t>(tot);
        const int64_t c = ctx->gcount[w];
        if (c > 0 && c <= thr) {
            tot += static_cast<uint64_t>(std::min<int64_t>(c, K));
            ++nsp;
        }
        if (tot >= 0xFFFFFFF0ull) return LDA_OK;  // beyond 32-bit offsets: dense tables only
    }
    off[V] = static_cast<uint32_t>(tot);
    if (nsp == 0) return LDA_OK;
    DA(S.sp_off, static_cast<size_t>(V) + 1);
    DA(S.sp_nnz, static_cast<size_t>(V));
    DA(S.sp_ent, 2 * static_cast<size_t>(tot));
    DA(S.s32, static_cast<size_t>((K + 3) & ~3));
    CU(cudaMemcpy(S.sp_off, off.data(), sizeof(uint32_t) * off.size(), cudaMemcpyHostToDevice));
    S.sp_words = nsp;
    S.sp_cap = static_cast<int64_t>(tot);
    return LDA_OK;
}

int ensure_events(lda_ctx *ctx, size_t n) {
    while (ctx->ev.size() < n) {
        cudaEvent_t e;
        CU(cudaEventCreate(&e));
        ctx->ev.push_back(e);
    }
    return LDA_OK;
}

// Rebuild n_wk, n_k (and allreduce them) and θ from tok_z.
int rebuild_counts(lda_ctx *ctx, int *launches) {
    lda::DevState &S = ctx->S;
    KL(lda::launch_recount(S, ctx->stream, launches));
    if (ctx->world > 1) {
        COMM(allreduce_i32(S.nwk, static_cast<size_t>(S.V) * S.K + S.K, ctx->stream, e_));
    }
    KL(lda::launch_theta(S, S.stat, ctx->stream, launches));
    unsigned long long hs[2] = {0, 0};
    CU(cudaMemcpyAsync(hs, S.stat, sizeof(hs), cudaMemcpyDeviceToHost, ctx->stream));
    CU(cudaStreamSynchronize(ctx->stream));
    ctx->cur_lnnz = static_cast<int64_t>(hs[0]);
    ctx->cur_nnz = static_cast<int64_t>(hs[1]);
    return LDA_OK;
}


// ---------------------------------------------------------------------------
// f3: out-of-HBM streaming (Alg. 1 WorkSchedule2, L835-859, §5.1)
// ---------------------------------------------------------------------------
// The device view of chunk m in slot sl: the configured kernels and model
// buffers of ctx->S, the chunk's resident tables, the slot's token buffers.
lda::DevState chunk_view(lda_ctx *ctx, int64_t m, int sl) {
    const lda_stream::Chunk &c = *ctx->chunks[m];
    const lda_stream::Slot &b = ctx->slot[sl];
    lda::DevState v = ctx->S;
    v.D = c.D;
    v.T = c.T;
    v.ntiles = c.H.ntiles;
    v.rows32 = c.H.rows32;
    v.doc_ptr32 = c.R.doc_ptr32;
    v.row_off32 = c.R.row_off32;
    v.segs = c.R.segs;
    v.rchunks = c.R.rchunks;
    v.n_rchunks = c.R.n_rchunks;
    v.split_words = nullptr;
    v.n_split = 0;
    v.titems = c.R.titems;
    v.n_titems = c.R.n_titems;
    v.cbase = c.R.cbase;
    v.tok_row = b.tok_row;
    v.doc_map = b.doc_map;
    v.tok_z = b.z;
    v.z_doc = b.z_doc;
    v.rows = b.rows;
    return v;
}

// DataTransfer(Chunk, θ: CPU -> GPU) of Alg. 1 lines 26-27
int chunk_h2d(lda_ctx *ctx, int64_t m, int sl, cudaStream_t st, bool with_z) {
    const lda_stream::Chunk &c = *ctx->chunks[m];
    const lda_stream::Slot &b = ctx->slot[sl];
    const size_t T = static_cast<size_t>(c.T);
    if (T) {
        CU(cudaMemcpyAsync(b.tok_row, c.H.tok_row.data(), 4 * T, cudaMemcpyHostToDevice, st));
        CU(cudaMemcpyAsync(b.doc_map, c.H.doc_map.data(), 4 * T, cudaMemcpyHostToDevice, st));
        if (with_z) CU(cudaMemcpyAsync(b.z, c.hz, 2 * T, cudaMemcpyHostToDevice, st));
    }
    CU(cudaMemcpyAsync(b.rows, c.hrows, 32 * c.H.rows32, cudaMemcpyHostToDevice, st));
    return LDA_OK;
}

// DataTransfer(θ: GPU -> CPU) of Alg. 1 line 29 (and the chunk's new z)
int chunk_d2h(lda_ctx *ctx, int64_t m, int sl, cudaStream_t st) {
    const lda_stream::Chunk &c = *ctx->chunks[m];
    const lda_stream::Slot &b = ctx->slot[sl];
    if (c.T) CU(cudaMemcpyAsync(c.hz, b.z, 2 * static_cast<size_t>(c.T), cudaMemcpyDeviceToHost, st));
    CU(cudaMemcpyAsync(c.hrows, b.rows, 32 * c.H.rows32, cudaMemcpyDeviceToHost, st));
    return LDA_OK;
}

// n_wk, n_k (accumulated over the chunks, then exchanged) and every chunk's θ
// from z; init = true draws the random initial z first (t = 0, X10).
int chunked_rebuild(lda_ctx *ctx, bool init, int *launches) {
    lda::DevState &S = ctx->S;
    const size_t nwk_n = static_cast<size_t>(S.V) * S.K + S.K;
    CU(cudaMemsetAsync(S.nwk, 0, nwk_n * sizeof(int32_t), ctx->stream));
    int64_t lnnz = 0, nnz = 0;
    for (int64_t m = 0; m < static_cast<int64_t>(ctx->chunks.size()); ++m) {
        int r = chunk_h2d(ctx, m, 0, ctx->stream, !init);
        if (r != LDA_OK) return r;
        lda::DevState v = chunk_view(ctx, m, 0);
        if (init) KL(lda::launch_init(v, ctx->stream));
        KL(lda::launch_recount(v, ctx->stream, launches, 0, -1, false));
        KL(lda::launch_theta(v, S.stat, ctx->stream, launches));
        r = chunk_d2h(ctx, m, 0, ctx->stream);
        if (r != LDA_OK) return r;
        unsigned long long hs[2] = {0, 0};
        CU(cudaMemcpyAsync(hs, S.stat, sizeof(hs), cudaMemcpyDeviceToHost, ctx->stream));
        CU(cudaStreamSynchronize(ctx->stream));
        lnnz += static_cast<int64_t>(hs[0]);
        nnz += static_cast<int64_t>(hs[1]);
    }
    if (ctx->world > 1) COMM(allreduce_i32(S.nwk, nwk_n, ctx->stream, e_));
    CU(cudaStreamSynchronize(ctx->stream));
    ctx->cur_lnnz = lnnz;
    ctx->cur_nnz = nnz;
    return LDA_OK;
}

int load_chunked(lda_ctx *ctx, const int64_t *doc_ptr, const int32_t *words, int64_t Dg, int64_t Tg,
                 const std::vector<int64_t> &cbase_rank, uint64_t seed) {
    lda::DevState &S = ctx->S;
    const int32_t V = ctx->V, K = ctx->K;
    const int64_t M = std::max<int64_t>(1, std::min<int64_t>(ctx->stream_chunks, std::max<int64_t>(Dg, 1)));
    std::vector<int64_t> bounds(M + 1);
    if (lda_partition_docs(Dg, doc_ptr, static_cast<int32_t>(M), bounds.data()) != LDA_OK)
        return fail(ctx, LDA_EINVAL, "chunk partition failed");
    const int64_t kscale = S.sweep_tile_cta ? std::max<int64_t>(1, K / 1024) : 1;
    int l2 = 0;
    CU(cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, ctx->device));
    std::vector<int64_t> seen(V, 0);
    size_t max_T = 1, max_rows32 = 4;
    for (int64_t m = 0; m < M; ++m) {
        auto c = std::make_unique<lda_stream::Chunk>();
        const int64_t d0 = bounds[m], d1 = bounds[m + 1], t0 = doc_ptr[d0], t1 = doc_ptr[d1];
        c->doc_begin = d0;
        c->D = d1 - d0;
        c->tok_begin = t0;
        c->T = t1 - t0;
        std::vector<int64_t> dp(c->D + 1);
        for (int64_t d = 0; d <= c->D; ++d) dp[d] = doc_ptr[d0 + d] - t0;
        std::vector<int64_t> wc(V, 0), cb(V);
        lda::word_histogram(words + t0, c->T, V, ctx->threads, wc.data());
        // canonical bases: the chunk's tokens of word w follow those of the
        // rank's earlier chunks (documents stay in order, X18)
        for (int32_t w = 0; w < V; ++w) {
            cb[w] = cbase_rank[w] + seen[w];
            seen[w] += wc[w];
        }
        uint64_t r32 = 4;
        for (int64_t d = 0; d < c->D; ++d)
            r32 += 4 * static_cast<uint64_t>((std::min<int64_t>(dp[d + 1] - dp[d], K) + 1 + 31) / 32);
        int64_t tile = ctx->tile_tokens;
        if (tile < 0) {
            const double target = 0.5 * static_cast<double>(l2 > 0 ? l2 : (126 << 20));
            tile = 32.0 * r32 <= target ? 0
                                         : std::max<int64_t>(int64_t(1) << 20,
                                                             static_cast<int64_t>(c->T * (target / (32.0 * r32))));
        }
        std::string e = lda::build_layout(dp.data(), words + t0, c->D, V, K, cb.data(), tile,
                                          ctx->chunk_tokens, ctx->recount_tokens, ctx->threads, 2,
                                          ctx->tail_per_tile * kscale, c->H, {}, wc.data(), /*host_tok_row=*/true);
        if (!e.empty()) return fail(ctx, LDA_ERANGE, e);
        lda::HostLayout &H = c->H;
        // every chunk adds into the same n_wk rows: all recount items accumulate
        for (auto &rc : H.rchunks) rc.word |= 0x80000000u;
        // page-lock the streamed host tables (async DataTransfer)
        if (c->T) {
            CU(cudaHostRegister(H.tok_row.data(), 4 * static_cast<size_t>(c->T), cudaHostRegisterDefault));
            cudaError_t ce = cudaHostRegister(H.doc_map.data(), 4 * static_cast<size_t>(c->T), cudaHostRegisterDefault);
            if (ce != cudaSuccess) {
                cudaHostUnregister(H.tok_row.data());
                return fail(ctx, LDA_ECUDA, std::string("cudaHostRegister: ") + cudaGetErrorString(ce));
            }
            c->registered = true;
        }
        CU(cudaMallocHost(&c->hz, 2 * std::max<size_t>(1, c->T)));
        CU(cudaMallocHost(&c->hrows, 32 * H.rows32));
        std::memset(c->hrows, 0, 32 * H.rows32);
        lda::DevState &R = c->R;
        DA(R.doc_ptr32, c->D + 1);
        DA(R.row_off32, std::max<int64_t>(c->D, 1));
        DA(R.segs, H.segs.size());
        DA(R.rchunks, H.rchunks.size());
        DA(R.titems, H.titems.size());
        DA(R.cbase, V);
        R.n_rchunks = static_cast<int64_t>(H.rchunks.size());
        R.n_titems = static_cast<int64_t>(H.titems.size());
        std::vector<uint64_t> cb64(cb.begin(), cb.end());
        CU(cudaMemcpy(R.doc_ptr32, H.doc_ptr32.data(), 4 * (c->D + 1), cudaMemcpyHostToDevice));
        if (c->D) CU(cudaMemcpy(R.row_off32, H.row_off32.data(), 4 * c->D, cudaMemcpyHostToDevice));
        if (!H.segs.empty())
            CU(cudaMemcpy(R.segs, H.segs.data(), sizeof(lda::Seg) * H.segs.size(), cudaMemcpyHostToDevice));
        if (!H.rchunks.empty())
            CU(cudaMemcpy(R.rchunks, H.rchunks.data(), sizeof(lda::RecountChunk) * H.rchunks.size(),
                          cudaMemcpyHostToDevice));
        if (!H.titems.empty())
            CU(cudaMemcpy(R.titems, H.titems.data(), sizeof(lda::TileItem) * H.titems.size(), cudaMemcpyHostToDevice));
        CU(cudaMemcpy(R.cbase, cb64.data(), 8 * static_cast<size_t>(V), cudaMemcpyHostToDevice));
        max_T = std::max<size_t>(max_T, static_cast<size_t>(c->T));
        max_rows32 = std::max<size_t>(max_rows32, H.rows32);
        ctx->chunks.push_back(std::move(c));
    }
    // two device slots (chunk m+1's transfer overlaps chunk m's sweep) and the
    // resident model
    for (auto &b : ctx->slot) {
        DA(b.tok_row, max_T);
        DA(b.doc_map, max_T);
        DA(b.z, max_T + 8);
        DA(b.z_doc, max_T + 8);
        DA(b.rows, 8 * max_rows32);
        CU(cudaEventCreateWithFlags(&b.in, cudaEventDisableTiming));
        CU(cudaEventCreateWithFlags(&b.done, cudaEventDisableTiming));
        CU(cudaEventCreateWithFlags(&b.free_, cudaEventDisableTiming));
    }
    CU(cudaStreamCreateWithFlags(&ctx->h2d_stream, cudaStreamNonBlocking));
    CU(cudaStreamCreateWithFlags(&ctx->d2h_stream, cudaStreamNonBlocking));
    for (auto &b : ctx->slot) CU(cudaEventRecord(b.free_, ctx->d2h_stream));
    const size_t nwk_n = static_cast<size_t>(V) * K + K;
    DA(S.nwk, nwk_n);
    DA(S.nwk_alt, nwk_n);
    DA(S.wtab, S.wt_bytes * static_cast<size_t>(V));
    DA(S.denom, K);
    DA(S.counter, 4);
    DA(S.stat, 4);
    DA(S.ll_part, 2 * S.ll_blocks + 2);
    DA(S.ll_out, 2);
    S.V = V;
    S.K = K;
    S.D = Dg;
    S.T = Tg;
    S.alpha = ctx->alpha;
    S.beta = ctx->beta;
    S.seed = seed;
    S.ntiles = 0;
    for (auto &c : ctx->chunks) S.ntiles += c->H.ntiles;
    {
        const int rs = setup_sparse_rows(ctx);
        if (rs != LDA_OK) return rs;
    }
    int launches = 0;
    int r = chunked_rebuild(ctx, true, &launches);
    if (r != LDA_OK) return r;
    ctx->loaded = true;
    ctx->sweeps = 0;
    ctx->stats.local_tokens = Tg;
    ctx->stats.local_docs = Dg;
    ctx->stats.global_tokens = ctx->T_global;
    ctx->stats.world = ctx->world;
    int64_t items = 0;
    for (auto &c : ctx->chunks) items += c->R.n_titems;
    ctx->stats.n_sample_chunks = items;
    ctx->stats.tile_tokens = ctx->tile_tokens_used;
    ctx->stats.n_tiles = S.ntiles;
    ctx->stats.sampler = S.sweep_tile ? 2 : 3;
    ctx->stats.n_stream_chunks = M;
    ctx->stats.n_sparse_words = S.sp_words;
    ctx->stats.sum_nnz_doc = ctx->cur_nnz;
    return LDA_OK;
}

// One sweep over M streamed chunks (Alg. 1 lines 24-33): per-word tables once,
// then for every chunk: H2D (h2d stream) -> sample + recount into the next
// n_wk + θ rebuild (compute stream) -> D2H of z and θ (d2h stream), two slots
// in flight; then the exchange of the accumulated counts.  E: the sweep's 8
// events; stat: 2·M θ statistics of the sweep.
int sweep_chunked(lda_ctx *ctx, uint32_t t, cudaEvent_t *E, unsigned long long *stat, int *launches) {
    lda::DevState &S = ctx->S;
    const size_t nwk_n = static_cast<size_t>(S.V) * S.K + S.K;
    CU(cudaEventRecord(E[0], ctx->stream));
    KL(lda::launch_sweep(S, t, ctx->stream, launches, E[6], 1));  // prologue + word tables (a2, a3)
    CU(cudaMemsetAsync(S.nwk_alt, 0, nwk_n * sizeof(int32_t), ctx->stream));
    const int64_t M = static_cast<int64_t>(ctx->chunks.size());
    for (int64_t m = 0; m < M; ++m) {
        const int sl = static_cast<int>(m & 1);
        lda_stream::Slot &b = ctx->slot[sl];
        CU(cudaStreamWaitEvent(ctx->h2d_stream, b.free_, 0));  // the slot's previous chunk is back on the host
        int r = chunk_h2d(ctx, m, sl, ctx->h2d_stream, true);
        if (r != LDA_OK) return r;
        CU(cudaEventRecord(b.in, ctx->h2d_stream));
        CU(cudaStreamWaitEvent(ctx->stream, b.in, 0));
        lda::DevState v = chunk_view(ctx, m, sl);
        KL(lda::launch_sweep(v, t, ctx->stream, launches, nullptr, 2));  // a4 against the frozen n_wk
        lda::DevState vr = v;
        vr.nwk = S.nwk_alt;                                              // ϕ update: accumulate
        KL(lda::launch_recount(vr, ctx->stream, launches, 0, -1, false));
        KL(lda::launch_theta(v, stat + 2 * m, ctx->stream, launches));   // a5
        CU(cudaEventRecord(b.done, ctx->stream));
        CU(cudaStreamWaitEvent(ctx->d2h_stream, b.done, 0));
        r = chunk_d2h(ctx, m, sl, ctx->d2h_stream);
        if (r != LDA_OK) return r;
        CU(cudaEventRecord(b.free_, ctx->d2h_stream));
    }
    std::swap(S.nwk, S.nwk_alt);
    CU(cudaEventRecord(E[1], ctx->stream));
    CU(cudaEventRecord(E[2], ctx->stream));
    CU(cudaEventRecord(E[3], ctx->stream));
    if (ctx->world > 1) {
        CU(cudaStreamWaitEvent(ctx->comm_stream, E[2], 0));
        CU(cudaEventRecord(E[7], ctx->comm_stream));
        COMM(allreduce_i32(S.nwk, nwk_n, ctx->comm_stream, e_));
        CU(cudaEventRecord(E[4], ctx->comm_stream));
        CU(cudaStreamWaitEvent(ctx->stream, E[4], 0));
    }
    CU(cudaEventRecord(E[5], ctx->stream));
    return LDA_OK;
}

// LL over the chunks: the word part once (rank 0), the doc part chunk by chunk
int chunked_loglik(lda_ctx *ctx, double h[2]) {
    h[0] = h[1] = 0.0;
    CU(cudaStreamSynchronize(ctx->d2h_stream));
    for (int64_t m = 0; m < static_cast<int64_t>(ctx->chunks.size()); ++m) {
        const lda_stream::Chunk &c = *ctx->chunks[m];
        CU(cudaMemcpyAsync(ctx->slot[0].rows, c.hrows, 32 * c.H.rows32, cudaMemcpyHostToDevice, ctx->stream));
        lda::DevState v = chunk_view(ctx, m, 0);
        int launches = 0;
        KL(lda::launch_loglik(v, m == 0 && ctx->rank == 0, ctx->stream, &launches));
        double p[2];
        CU(cudaMemcpyAsync(p, ctx->S.ll_out, sizeof(p), cudaMemcpyDeviceToHost, ctx->stream));
        CU(cudaStreamSynchronize(ctx->stream));
        h[0] += p[0];
        h[1] += p[1];
    }
    return LDA_OK;
}

// LL sums (word part, doc part) of the current state, summed over the ranks
int loglik_pair(lda_ctx *ctx, double h[2]) {
    lda::DevState &S = ctx->S;
    if (!ctx->chunks.empty()) {
        int r = chunked_loglik(ctx, h);
        if (r != LDA_OK) return r;
        if (ctx->world > 1) {
            CU(cudaMemcpyAsync(S.ll_out, h, 2 * sizeof(double), cudaMemcpyHostToDevice, ctx->stream));
            COMM(allreduce_f64(S.ll_out, 2, ctx->stream, e_));
            CU(cudaMemcpyAsync(h, S.ll_out, 2 * sizeof(double), cudaMemcpyDeviceToHost, ctx->stream));
        }
        CU(cudaStreamSynchronize(ctx->stream));
        return LDA_OK;
    }
    int launches = 0;
    KL(lda::launch_loglik(S, ctx->rank == 0, ctx->stream, &launches));
    if (ctx->world > 1) COMM(allreduce_f64(S.ll_out, 2, ctx->stream, e_));
    CU(cudaMemcpyAsync(h, S.ll_out, 2 * sizeof(double), cudaMemcpyDeviceToHost, ctx->stream));
    CU(cudaStreamSynchronize(ctx->stream));
    return LDA_OK;
}

// option loglik_every: the LL after sweep t, outside the sweep's events (X23)
int log_loglik(lda_ctx *ctx, uint32_t t, std::vector<int64_t> &ll_at) {
    if (ctx->loglik_every <= 0 || t % static_cast<uint64_t>(ctx->loglik_every) != 0) return LDA_OK;
    double h[2];
    int r = loglik_pair(ctx, h);
    if (r != LDA_OK) return r;
    ll_at.push_back(static_cast<int64_t>(t));
    ctx->ll_pending.push_back(h[0] + h[1]);
    return LDA_OK;
}

}  // namespace

extern "C" {

const char *lda_version(void) { return "lda-b200 0.1 (sm_100a)"; }

const char *lda_last_error(const lda_ctx *ctx) {
    if (!ctx) return "null context";
    return ctx->err.c_str();
}

int lda_create(int64_t D, int32_t V, int32_t K, double alpha, double beta, lda_ctx **out) {
    if (!out) return LDA_EINVAL;
    *out = nullptr;
    if (D < 1 || V < 1 || K < 1 || K > 65536) return LDA_EINVAL;
    if (!std::isfinite(alpha) || !std::isfinite(beta) || !(alpha > 0) || !(beta > 0)) return LDA_EINVAL;
    if (K > kMaxK) return LDA_ERANGE;
    lda_ctx *c = new (std::nothrow) lda_ctx();
    if (!c) return LDA_ENOMEM;
    c->D = D;
    c->V = V;
    c->K = K;
    c->alpha = alpha;
    c->beta = beta;
    *out = c;
    return LDA_OK;
}

int lda_set_option(lda_ctx *ctx, const char *key, int64_t value) {
    PRECHECK(ctx);
    if (!key) return fail(ctx, LDA_EINVAL, "null option key");
    if (ctx->loaded) return fail(ctx, LDA_ESTATE, "options must be set before lda_load_corpus");
    std::string k(key);
    if (k == "device") {
        if (value < 0 || value > 1024) return fail(ctx, LDA_EINVAL, "bad device");
        ctx->device = static_cast<int>(value);
    } else if (k == "exclude_self") {
        if (value != 0 && value != 1) return fail(ctx, LDA_EINVAL, "exclude_self must be 0 or 1");
        ctx->exclude_self = static_cast<int>(value);
    } else if (k == "chunk_tokens") {
        if (value < 32 || value > (int64_t(1) << 30)) return fail(ctx, LDA_EINVAL, "chunk_tokens out of range");
        ctx->chunk_tokens = value;
    } else if (k == "recount_tokens") {
        if (value < 256 || value > (int64_t(1) << 31)) return fail(ctx, LDA_EINVAL, "recount_tokens out of range");
        ctx->recount_tokens = value;
    } else if (k == "tile_tokens") {
        if (value < -1) return fail(ctx, LDA_EINVAL, "tile_tokens must be -1 (auto) or >= 0");
        ctx->tile_tokens = value;
    } else if (k == "sampler") {
        if (value != -1 && value != 0 && value != 2 && value != 3)
            return fail(ctx, LDA_EINVAL, "sampler must be -1 (auto), 0, 2 or 3");
        ctx->sampler = static_cast<int>(value);
    } else if (k == "tail_per_tile") {
        if (value < 0 || value > (int64_t(1) << 30)) return fail(ctx, LDA_EINVAL, "tail_per_tile out of range");
        ctx->tail_per_tile = value;
    } else if (k == "fused_recount") {
        if (value != 0 && value != 1) return fail(ctx, LDA_EINVAL, "fused_recount must be 0 or 1");
        ctx->fused_recount = static_cast<int>(value);
    } else if (k == "certify_slack") {
        if (value < 1 || value > (int64_t(1) << 40)) return fail(ctx, LDA_EINVAL, "certify_slack out of range");
        ctx->certify_slack = value;
    } else if (k == "stream_chunks") {
        if (value < 1 || value > 4096) return fail(ctx, LDA_EINVAL, "stream_chunks must be in [1, 4096]");
        ctx->stream_chunks = value;
    } else if (k == "comm_pipeline") {
        if (value < 1 || value > 64) return fail(ctx, LDA_EINVAL, "comm_pipeline must be in [1, 64]");
        ctx->comm_pipeline = value;
    } else if (k == "sparse_words") {
        if (value < -1) return fail(ctx, LDA_EINVAL, "sparse_words must be -1 (auto), 0 (off) or > 0");
        ctx->sparse_words = value;
    } else if (k == "loglik_every") {
        if (value < 0 || value > (int64_t(1) << 31)) return fail(ctx, LDA_EINVAL, "loglik_every must be >= 0");
        ctx->loglik_every = value;
    } else if (k == "threads") {
        if (value < 0 || value > 1024) return fail(ctx, LDA_EINVAL, "threads out of range");
        ctx->threads = static_cast<int>(value);
    } else {
        return fail(ctx, LDA_EINVAL, "unknown option '" + k + "'");
    }
    return LDA_OK;
}

int lda_nccl_unique_id(void *out128) {
    if (!out128) return LDA_EINVAL;
    std::string err;
    return lda::nccl_unique_id(out128, err);
}

int lda_init_dist(lda_ctx *ctx, int32_t rank, int32_t world, const void *uid) {
    PRECHECK(ctx);
    if (ctx->loaded || ctx->comm) return fail(ctx, LDA_ESTATE, "lda_init_dist must precede lda_load_corpus");
    if (world < 1 || rank < 0 || rank >= world) return fail(ctx, LDA_EINVAL, "bad rank/world");
    if (world == 1) {
        ctx->rank = 0;
        ctx->world = 1;
        return LDA_OK;
    }
    if (!uid) return fail(ctx, LDA_EINVAL, "null nccl unique id");
    std::string err;
    int r = lda::make_nccl_comm(rank, world, uid, ctx->device, ctx->comm, err);
    if (r != LDA_OK) return fail(ctx, r, err);
    ctx->rank = rank;
    ctx->world = world;
    return LDA_OK;
}

int lda_peer_group_create(int32_t world, lda_peer_group **out) {
    if (!out) return LDA_EINVAL;
    *out = nullptr;
    if (world < 1 || world > lda::kMaxPeers) return LDA_EINVAL;
    lda_peer_group *h = new (std::nothrow) lda_peer_group();
    if (!h) return LDA_ENOMEM;
    h->g = std::make_shared<lda::PeerGroup>(world);
    *out = h;
    return LDA_OK;
}

void lda_peer_group_destroy(lda_peer_group *g) { delete g; }

int lda_init_peer(lda_ctx *ctx, lda_peer_group *g, int32_t rank) {
    PRECHECK(ctx);
    if (ctx->loaded || ctx->comm) return fail(ctx, LDA_ESTATE, "lda_init_peer must precede lda_load_corpus");
    if (!g || !g->g) return fail(ctx, LDA_EINVAL, "null peer group");
    std::string err;
    int r = lda::make_peer_comm(g->g, rank, ctx->device, ctx->comm, err);
    if (r != LDA_OK) return fail(ctx, r, err);
    ctx->rank = rank;
    ctx->world = g->g->world();
    return LDA_OK;
}

int lda_canonical_bases(int32_t V, int32_t world, int32_t rank, const int64_t *word_counts, int64_t *cbase,
                        int64_t *total) {
    if (V < 1 || world < 1 || rank < 0 || rank >= world || !word_counts || !cbase) return LDA_EINVAL;
    int64_t run = 0;
    for (int32_t w = 0; w < V; ++w) {
        int64_t before_rank = 0, tot = 0;
        for (int32_t g = 0; g < world; ++g) {
            const int64_t n = word_counts[static_cast<size_t>(g) * V + w];
            if (n < 0) return LDA_EINVAL;
            if (g < rank) before_rank += n;
            tot += n;
        }
        cbase[w] = run + before_rank;
        run += tot;
    }
    if (total) *total = run;
    return LDA_OK;
}

int lda_partition_docs(int64_t D, const int64_t *doc_ptr, int32_t world, int64_t *doc_begin) {
    if (D < 0 || !doc_ptr || world < 1 || !doc_begin) return LDA_EINVAL;
    if (doc_ptr[0] != 0) return LDA_EINVAL;
    for (int64_t d = 0; d < D; ++d)
        if (doc_ptr[d + 1] < doc_ptr[d]) return LDA_EINVAL;
    const int64_t T = doc_ptr[D];
    doc_begin[0] = 0;
    for (int32_t g = 1; g < world; ++g) {
        // first d with doc_ptr[d] >= ceil(g*T/world)   (X21)
        const __int128 num = static_cast<__int128>(g) * T;
        const int64_t target = static_cast<int64_t>((num + world - 1) / world);
        const int64_t *it = std::lower_bound(doc_ptr, doc_ptr + D + 1, target);
        int64_t d = it - doc_ptr;
        doc_begin[g] = std::min(std::max(d, doc_begin[g - 1]), D);
    }
    doc_begin[world] = D;
    return LDA_OK;
}

int lda_load_corpus(lda_ctx *ctx, int64_t doc_begin, int64_t doc_end, const int64_t *doc_ptr,
                    const int32_t *words, uint64_t seed) {
    PRECHECK(ctx);
    if (ctx->loaded) return fail(ctx, LDA_ESTATE, "corpus already loaded");
    if (doc_begin < 0 || doc_end < doc_begin || doc_end > ctx->D)
        return fail(ctx, LDA_EINVAL, "document range outside [0, D]");
    if (ctx->world == 1 && (doc_begin != 0 || doc_end != ctx->D))
        return fail(ctx, LDA_EINVAL, "with world == 1 the whole corpus [0, D) must be loaded");
    const int64_t Dg = doc_end - doc_begin;
    bool range_err = false;
    lda::tmark(nullptr);
    const auto load_t0 = std::chrono::steady_clock::now();
    // the CUDA setup (streams, kernel configuration: the process's first
    // kernel-attribute calls load the module, ~80 ms) runs in a helper thread
    // while the host validates the words
    lda::DevState &S = ctx->S;
    S.K = ctx->K;
    S.exclude_self = ctx->exclude_self;
    S.sampler = ctx->sampler;
    S.certify_slack = static_cast<double>(ctx->certify_slack);
    S.tile_fused = ctx->fused_recount != 0 && ctx->stream_chunks == 1;  // chunks: the recount kernel accumulates
    cudaError_t setup_err = cudaSuccess;
    std::thread setup([&] {
        cudaError_t e = cudaSetDevice(ctx->device);
        if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&ctx->stream, cudaStreamNonBlocking);
        if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&ctx->comm_stream, cudaStreamNonBlocking);
        if (e == cudaSuccess) e = static_cast<cudaError_t>(lda::configure_kernels(S));
        setup_err = e;
    });
    // the document offsets first; the words (one pass: validation + the
    // local word histogram) here too unless the layout's own per-tile count
    // pass does both (one rank, tile samplers, resident corpus)
    std::vector<int64_t> local(ctx->V, 0);
    std::string v = lda::validate_corpus(doc_ptr, words, Dg, ctx->V, &range_err, nullptr, ctx->threads, false);
    setup.join();
    if (!v.empty()) return fail(ctx, range_err ? LDA_ERANGE : LDA_EINVAL, v);
    if (setup_err != cudaSuccess) {
        // an invalid corpus is reported as such even without a device
        v = lda::validate_corpus(doc_ptr, words, Dg, ctx->V, &range_err, nullptr, ctx->threads);
        if (!v.empty()) return fail(ctx, range_err ? LDA_ERANGE : LDA_EINVAL, v);
        return fail(ctx, LDA_ECUDA, std::string("CUDA setup: ") + cudaGetErrorString(setup_err));
    }
    const bool words_in_layout = ctx->world == 1 && ctx->stream_chunks == 1 && (S.sweep_tile || S.sweep_tile_cta);
    if (!words_in_layout) {
        v = lda::validate_corpus(doc_ptr, words, Dg, ctx->V, &range_err, local.data(), ctx->threads);
        if (!v.empty()) return fail(ctx, range_err ? LDA_ERANGE : LDA_EINVAL, v);
    }
    lda::tmark("validate (+ word histogram) || CUDA setup");
    const int64_t Tg = doc_ptr[Dg];
    // θ row storage: 128-byte aligned rows of min(L_d, K) + 1 words, in
    // 32-byte units (the layout's row_off32; checked against H.rows32 after
    // the layout).  Its range is checked here, before any allocation.
    uint64_t r32 = 4;
    for (int64_t d = 0; d < Dg; ++d)
        r32 += 4 * static_cast<uint64_t>((std::min<int64_t>(doc_ptr[d + 1] - doc_ptr[d], ctx->K) + 1 + 31) / 32);
    if (r32 >= (uint64_t(1) << 32) - 60) return fail(ctx, LDA_ERANGE, "θ row storage exceeds 2^32 x 32 bytes");
    const int32_t V = ctx->V, K = ctx->K;

    CU(cudaSetDevice(ctx->device));

    // Local word histogram -> canonical bases.  c for rank g's tokens of word
    // w starts at Σ_{w'<w} T(w') + Σ_{g'<g} T_{g'}(w)   (X18, §8(c) step 2).
    std::vector<int64_t> all(static_cast<size_t>(V) * ctx->world, 0);
    if (ctx->world > 1) {
        int64_t *d_all = nullptr;
        DA(d_all, all.size());
        CU(cudaMemcpyAsync(d_all + static_cast<size_t>(ctx->rank) * V, local.data(), sizeof(int64_t) * V,
                           cudaMemcpyHostToDevice, ctx->stream));
        COMM(allgather_i64(d_all + static_cast<size_t>(ctx->rank) * V, d_all, V, ctx->stream, e_));
        CU(cudaMemcpyAsync(all.data(), d_all, sizeof(int64_t) * all.size(), cudaMemcpyDeviceToHost, ctx->stream));
        CU(cudaStreamSynchronize(ctx->stream));
    } else {
        std::copy(local.begin(), local.end(), all.begin());
    }
    std::vector<int64_t> cbase(V);
    if (!words_in_layout) {
        int64_t run = 0;
        lda_canonical_bases(V, ctx->world, ctx->rank, all.data(), cbase.data(), &run);
        ctx->T_global = run;
        ctx->gcount.assign(V, 0);
        for (int32_t g = 0; g < ctx->world; ++g)
            for (int32_t w = 0; w < V; ++w) ctx->gcount[w] += all[static_cast<size_t>(g) * V + w];
    }

    lda::HostLayout &H = ctx->H;
    // the per-token tables go to the device tile by tile, copied by a helper
    // thread while the host prepares the next tile
    const bool tile_layout = S.sweep_tile || S.sweep_tile_cta;
    // the tile samplers' line tables flag a row's first line in bit 31
    if (tile_layout && r32 >= (uint64_t(1) << 31) - 60)
        return fail(ctx, LDA_ERANGE,
                    "θ row storage exceeds 2^31 x 32 bytes (64 GB) on one rank: use more ranks or sampler 0");
    // tiles (Alg. 1 WorkSchedule1's resident shard, sampled tile by tile):
    // auto = tiles whose θ rows fill about half the L2, so that a tile's rows
    // are read from HBM about once per sweep
    int64_t tile_tokens = ctx->tile_tokens;
    if (tile_tokens < 0) {
        int l2 = 0;
        CU(cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, ctx->device));
        const double target = 0.5 * static_cast<double>(l2 > 0 ? l2 : (126 << 20));
        const double row_bytes = 32.0 * static_cast<double>(r32);
        tile_tokens = row_bytes <= target ? 0
                                          : std::max<int64_t>(int64_t(1) << 20,
                                                              static_cast<int64_t>(Tg * (target / row_bytes)));
    }
    ctx->tile_tokens_used = tile_tokens;
    lda::tmark("histogram, streams, configure");
    if (ctx->stream_chunks > 1) {
        if (!tile_layout)
            return fail(ctx, LDA_EINVAL, "stream_chunks > 1 needs a tile sampler (2 or 3) and exclude_self = 0");
        return load_chunked(ctx, doc_ptr, words, Dg, Tg, cbase, seed);
    }
    // The device buffers are allocated by the copier thread below while the
    // host builds the layout (cudaMalloc of ~10 GB takes ~0.3-0.5 s, all of
    // it otherwise on the load path): first the per-token tables it copies
    // into, then the large buffers that do not depend on the layout.
    std::vector<std::pair<void **, size_t>> pre;
    for (uint32_t **t : {&S.tok_row, &S.doc_map, tile_layout ? nullptr : &S.tok_crank})
        if (t) pre.push_back({reinterpret_cast<void **>(t), sizeof(uint32_t) * Tg});
    pre.push_back({reinterpret_cast<void **>(&S.tok_z), sizeof(uint16_t) * Tg});
    pre.push_back({reinterpret_cast<void **>(&S.z_doc), sizeof(uint16_t) * (Tg + 8)});
    const size_t nwk_bytes = sizeof(int32_t) * (static_cast<size_t>(V) * K + K);
    pre.push_back({reinterpret_cast<void **>(&S.nwk), nwk_bytes});
    if (S.sweep_fused) pre.push_back({reinterpret_cast<void **>(&S.nwk_alt), nwk_bytes});
    if (tile_layout) pre.push_back({reinterpret_cast<void **>(&S.wtab), S.wt_bytes * static_cast<size_t>(V)});
    std::vector<void *> pre_done;
    size_t pre_fail_bytes = 0;
    const uint64_t pre_rows32 = r32;
    struct Job {
        uint64_t p0, p1, t0, t1;
        int words = 0;  // 1: upload words[t0, t1) into S.tok_row (device layout: the sort's input)
    };
    std::vector<Job> jobs;
    std::mutex mu;
    std::condition_variable cv;
    bool jobs_done = false;
    cudaError_t copy_err = cudaSuccess;
    // the device buffers are allocated by copier 0; then all copiers move the
    // finished parts of the token tables (pageable host memory: the driver
    // stages each copy, so several copies run at once from several threads)
    const bool dev_scatter = tile_layout;  // doc_map built on the device (see below)
    bool words_pinned = false;
    int64_t words_left = 0;  // words upload jobs not finished (device layout)
    bool alloc_done = false;
    double copy_ms_total = 0.0, memcpy_ms_total = 0.0, alloc_ms = 0.0, alloc_arena_ms = 0.0, last_copy_end = 0.0,
           layout_end = 0.0;
    // page-locked staging ring: the copiers memcpy a finished piece of a token
    // table into a slot (in parallel, from several threads) and DMA it from
    // there -- the driver's own pageable path serialises the copies at ~10 GB/s
    constexpr int kCopiers = 4, kSlots = 8;
    constexpr size_t kSlotBytes = size_t(16) << 20;
    char *stage = nullptr;
    std::vector<int> free_slots;
    auto copier_main = [&](int id) {
        cudaSetDevice(ctx->device);
        cudaStream_t cs = nullptr;
        cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking);
        if (id == 0) {
            const auto c0 = std::chrono::steady_clock::now();
            cudaError_t err = cudaSuccess;
            // one allocation carved into the buffers (the per-call cost of
            // cudaMalloc, not the bytes, dominated: tens of ms per call)
            size_t total = 0;
            for (auto &pa : pre) total += (std::max<size_t>(pa.second, 1) + 511) & ~size_t(511);
            void *arena = nullptr;
            err = cudaMalloc(&arena, total);
            if (err != cudaSuccess) {
                pre_fail_bytes = total;
            } else {
                pre_done.push_back(arena);
                size_t off = 0;
                for (auto &pa : pre) {
                    *pa.first = static_cast<char *>(arena) + off;
                    off += (std::max<size_t>(pa.second, 1) + 511) & ~size_t(511);
                }
            }
            // (no staging ring when every copy is a straight DMA: the device
            // layout with page-locked words copies nothing else)
            const bool need_stage = !(dev_scatter && words_pinned);
            alloc_arena_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - c0).count();
            if (err == cudaSuccess && need_stage &&
                cudaHostAlloc(reinterpret_cast<void **>(&stage), kSlots * kSlotBytes, cudaHostAllocDefault) !=
                    cudaSuccess) {
                cudaGetLastError();
                stage = nullptr;  // fall back to pageable copies
            }
            std::lock_guard<std::mutex> lk(mu);
            if (err != cudaSuccess && copy_err == cudaSuccess) copy_err = err;
            if (stage)
                for (int k = 0; k < kSlots; ++k) free_slots.push_back(k);
            alloc_done = true;
            alloc_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - c0).count();
            cv.notify_all();
        }
        double copy_ms = 0.0, memcpy_ms = 0.0;
        for (;;) {
            Job j;
            {
                std::unique_lock<std::mutex> lk(mu);
                cv.wait(lk, [&] { return alloc_done && (!jobs.empty() || jobs_done); });
                if (jobs.empty()) break;
                j = jobs.front();
                jobs.erase(jobs.begin());
                if (copy_err != cudaSuccess) {  // drain the queue
                    if (j.words && --words_left == 0) cv.notify_all();
                    continue;
                }
            }
            const auto j0 = std::chrono::steady_clock::now();
            cudaError_t r = cudaSuccess;
            const size_t np = (j.p1 - j.p0) * sizeof(uint32_t), nt = (j.t1 - j.t0) * sizeof(uint32_t);
            // one piece of one table: through a staging slot when there is one
            auto put = [&](void *dst, const void *src, size_t bytes) {
                if (!bytes || r != cudaSuccess) return;
                int slot = -1;
                if (stage && bytes <= kSlotBytes) {
                    std::unique_lock<std::mutex> lk(mu);
                    cv.wait(lk, [&] { return !free_slots.empty(); });
                    slot = free_slots.back();
                    free_slots.pop_back();
                }
                if (slot < 0) {
                    r = cudaMemcpyAsync(dst, src, bytes, cudaMemcpyHostToDevice, cs);
                    if (r == cudaSuccess) r = cudaStreamSynchronize(cs);
                    return;
                }
                char *buf = stage + static_cast<size_t>(slot) * kSlotBytes;
                const auto m0 = std::chrono::steady_clock::now();
                std::memcpy(buf, src, bytes);
                memcpy_ms += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - m0).count();
                r = cudaMemcpyAsync(dst, buf, bytes, cudaMemcpyHostToDevice, cs);
                if (r == cudaSuccess) r = cudaStreamSynchronize(cs);
                std::lock_guard<std::mutex> lk(mu);
                free_slots.push_back(slot);
                cv.notify_all();
            };
            if (j.words) {
                // the words (device layout); straight DMA when the caller's buffer is page-locked
                if (words_pinned) {
                    r = cudaMemcpyAsync(S.tok_row + j.t0, words + j.t0, nt, cudaMemcpyHostToDevice, cs);
                    if (r == cudaSuccess) r = cudaStreamSynchronize(cs);
                } else {
                    put(S.tok_row + j.t0, words + j.t0, nt);
                }
            } else {
                if (H.tok_row.data()) put(S.tok_row + j.p0, H.tok_row.data() + j.p0, np);
                if (S.tok_crank) put(S.tok_crank + j.p0, H.tok_crank.data() + j.p0, np);
                put(S.doc_map + j.t0, H.doc_map.data() + j.t0, nt);
            }
            copy_ms += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - j0).count();
            if (r != cudaSuccess || j.words) {
                std::lock_guard<std::mutex> lk(mu);
                if (r != cudaSuccess && copy_err == cudaSuccess) copy_err = r;
                if (j.words && --words_left == 0) cv.notify_all();
            }
        }
        if (cs) cudaStreamDestroy(cs);
        std::lock_guard<std::mutex> lk(mu);
        copy_ms_total += copy_ms;
        memcpy_ms_total += memcpy_ms;
        last_copy_end = std::max(last_copy_end, std::chrono::duration<double, std::milli>(
                                                    std::chrono::steady_clock::now() - load_t0).count());
    };
    pre.push_back({reinterpret_cast<void **>(&S.rows), sizeof(uint32_t) * 8 * r32});
    // the device layout's scratch (see sorter_main), in the same allocation:
    // cudaMalloc / cudaFree on the sorter thread while the copiers and the
    // host pass run measured 1-150 ms and 1-820 ms
    uint32_t *sort_scratch = nullptr;
    const bool vtmp_rows = 8 * r32 >= static_cast<uint64_t>(Tg);
    const size_t sort_words = tile_layout && Tg > 0
                                  ? (vtmp_rows ? 0 : static_cast<size_t>(Tg)) + lda::radix_sort_temp_words(Tg) +
                                        2 * static_cast<size_t>(Dg + 1) + (static_cast<size_t>(V) + 3) / 4 + 64
                                  : 0;
    if (sort_words) pre.push_back({reinterpret_cast<void **>(&sort_scratch), sizeof(uint32_t) * sort_words});
    // the tile layout's doc-word map is built on the device (layout_gpu.cu):
    // the copiers upload the words into S.tok_row (rebuilt from doc_map
    // afterwards) while the host computes the counts
    if (dev_scatter && Tg > 0) {
        cudaPointerAttributes pa{};
        if (cudaPointerGetAttributes(&pa, words) == cudaSuccess)
            words_pinned = pa.type == cudaMemoryTypeHost;
        cudaGetLastError();
        const uint64_t piece = uint64_t(1) << 22;
        for (uint64_t t0 = 0; t0 < static_cast<uint64_t>(Tg); t0 += piece) {
            Job j{0, 0, t0, std::min<uint64_t>(static_cast<uint64_t>(Tg), t0 + piece)};
            j.words = 1;
            jobs.push_back(j);
            ++words_left;
        }
    }
    // The device layout (layout_gpu.cu: keys, stable radix sort, doc_map) runs
    // on a helper thread and its own stream as soon as the words are on the
    // device and the layout's first pass has fixed the tiles and the tail
    // words (on_keys), overlapping the rest of the host pass.
    bool keys_ready = false, sort_cancel = false, sort_range = false;
    cudaError_t sort_err = cudaSuccess;
    std::string sort_where;
    double sort_start_ms = 0.0, sort_end_ms = 0.0, sort_malloc_ms = 0.0, sort_kernels_ms = 0.0;
    auto sorter_main = [&]() {
        {
            std::unique_lock<std::mutex> lk(mu);
            cv.wait(lk, [&] { return sort_cancel || (keys_ready && alloc_done && words_left == 0); });
            if (sort_cancel || copy_err != cudaSuccess) return;
            sort_start_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - load_t0).count();
        }
        cudaError_t ce = cudaSetDevice(ctx->device);
        cudaStream_t ss = ctx->comm_stream;  // idle during the load
        // doc_map = the stable sort of the tokens by (tile, word)
        const uint64_t n = static_cast<uint64_t>(Tg);
        const int ndt = static_cast<int>(H.tile_doc.size()) - 1;
        const uint64_t maxkey = static_cast<uint64_t>(ndt + 1) * static_cast<uint64_t>(V);
        if (maxkey > 0xFFFFFFFFull) {
            sort_range = true;
            return;
        }
        int bits = 1;
        while (bits < 32 && (uint64_t(1) << bits) < maxkey) ++bits;
        // The sort's four T-word buffers are the load's own: the keys over the
        // words (S.tok_row), the keys' second buffer S.doc_map, the values in
        // the z buffers (S.tok_z, S.z_doc: >= 4·T contiguous bytes of the
        // arena) and the values' second buffer in the θ row storage when it
        // holds >= T words (zeroed after the load; else in sort_scratch).  The
        // final values land in the z buffers or the θ rows, never in doc_map,
        // which the inversion then writes.
        const size_t tw = lda::radix_sort_temp_words(n);
        uint32_t *tmp = sort_scratch;
        auto now_ms = [&] {
            return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - load_t0).count();
        };
        sort_malloc_ms = now_ms();
        uint32_t *keys = S.tok_row, *ktmp = S.doc_map, *vals = reinterpret_cast<uint32_t *>(S.tok_z);
        uint32_t *vtmp = vtmp_rows ? S.rows : tmp;
        uint32_t *rtmp = tmp + (vtmp_rows ? 0 : n);
        uint32_t *d_tile_doc = rtmp + tw;
        uint32_t *d_doc_ptr = d_tile_doc + H.tile_doc.size();
        uint8_t *d_tail = reinterpret_cast<uint8_t *>(d_doc_ptr + Dg + 1);
        bool in_tmp = false;
        int r = 0;
        ce = cudaMemcpyAsync(d_tile_doc, H.tile_doc.data(), sizeof(uint32_t) * H.tile_doc.size(),
                             cudaMemcpyHostToDevice, ss);
        if (ce == cudaSuccess)
            ce = cudaMemcpyAsync(d_doc_ptr, H.doc_ptr32.data(), sizeof(uint32_t) * (Dg + 1), cudaMemcpyHostToDevice, ss);
        if (ce == cudaSuccess) ce = cudaMemcpyAsync(d_tail, H.tail.data(), H.tail.size(), cudaMemcpyHostToDevice, ss);
        if (ce == cudaSuccess)
            r = lda::launch_layout_keys(d_doc_ptr, reinterpret_cast<const int32_t *>(S.tok_row), d_tail, d_tile_doc,
                                        ndt, V, Dg, keys, vals, S.num_sms, ss);
        if (ce == cudaSuccess && r == 0) r = lda::radix_sort_pairs(keys, vals, ktmp, vtmp, n, bits, rtmp, ss, &in_tmp);
        if (ce == cudaSuccess && r == 0) r = lda::launch_invert(in_tmp ? vtmp : vals, S.doc_map, n, ss);
        if (ce == cudaSuccess && r != 0) ce = static_cast<cudaError_t>(r);
        if (ce == cudaSuccess) ce = cudaStreamSynchronize(ss);
        sort_kernels_ms = now_ms();
        if (ce != cudaSuccess) {
            sort_err = ce;
            sort_where = "device layout";
            cudaGetLastError();
        }
        sort_end_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - load_t0).count();
    };
    std::thread sorter;
    if (dev_scatter && Tg > 0) sorter = std::thread(sorter_main);
    std::vector<std::thread> copiers;
    for (int id = 0; id < kCopiers; ++id) copiers.emplace_back(copier_main, id);
    auto on_final = [&](uint64_t p0, uint64_t p1, uint64_t t0, uint64_t t1) {
        {
            // in pieces of <= 4 M tokens (16 MB), so that the copiers share a tile
            std::lock_guard<std::mutex> lk(mu);
            const uint64_t piece = uint64_t(1) << 22;
            const uint64_t n = std::max<uint64_t>(1, std::max((p1 - p0 + piece - 1) / piece, (t1 - t0 + piece - 1) / piece));
            for (uint64_t q = 0; q < n; ++q)
                jobs.push_back(Job{p0 + (p1 - p0) * q / n, p0 + (p1 - p0) * (q + 1) / n, t0 + (t1 - t0) * q / n,
                                   t0 + (t1 - t0) * (q + 1) / n});
        }
        cv.notify_all();
    };
    // the large-K sampler copies a table of 4·K bytes per work item: words
    // with few tokens per tile go to the tail tile at a threshold scaled by
    // K/1024 (round 1, per-item tables: tiles scaled too, 1.94 -> 2.4 G
    // tokens/s at K = 8192); with CTA-shared tables the tiles themselves are
    // not scaled (5.31 -> 5.73 G tokens/s at NYTimes shape, K = 8192)
    const int64_t kscale = S.sweep_tile_cta ? std::max<int64_t>(1, K / 1024) : 1;
    std::string e = lda::build_layout(doc_ptr, words, Dg, V, K, cbase.data(), tile_tokens,
                                      ctx->chunk_tokens, ctx->recount_tokens, ctx->threads,
                                      tile_layout ? 2 : 0,
                                      ctx->tail_per_tile * kscale, H,
                                      on_final, words_in_layout ? nullptr : local.data(),
                                      /*host_tok_row=*/!tile_layout, /*device_scatter=*/dev_scatter, [&] {
                                          {
                                              std::lock_guard<std::mutex> lk(mu);
                                              keys_ready = true;
                                          }
                                          cv.notify_all();
                                      });
    {
        std::lock_guard<std::mutex> lk(mu);
        if (!keys_ready) sort_cancel = true;  // the layout failed before its first pass ended
        jobs_done = true;
        layout_end = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - load_t0).count();
    }
    cv.notify_all();
    for (auto &t : copiers) t.join();
    if (sorter.joinable()) sorter.join();
    if (stage) cudaFreeHost(stage);
    if (std::getenv("LDA_TIMING"))
        std::fprintf(stderr,
                     "[lda]   copiers: device allocation %.1f ms (arena %.1f), H2D %.1f ms (of which host memcpy %.1f; "
                     "summed over %d threads); layout end at %.1f ms, last copy end at %.1f ms (from the load start)\n",
                     alloc_ms, alloc_arena_ms, copy_ms_total, memcpy_ms_total, kCopiers, layout_end, last_copy_end);
    ctx->allocs.insert(ctx->allocs.end(), pre_done.begin(), pre_done.end());
    // a layout error (invalid word id, or a range) takes precedence over an allocation error
    if (!e.empty()) {
        cudaGetLastError();
        if (e.rfind("invalid: ", 0) == 0) return fail(ctx, LDA_EINVAL, e.substr(9));
        return fail(ctx, LDA_ERANGE, e);
    }
    if (words_in_layout) {
        // one rank: canonical bases from the layout's word counts (X18)
        int64_t run = 0;
        lda_canonical_bases(V, 1, 0, H.word_count.data(), cbase.data(), &run);
        ctx->T_global = run;
        ctx->gcount = H.word_count;
    }
    if (copy_err != cudaSuccess) {
        cudaGetLastError();
        return fail(ctx, copy_err == cudaErrorMemoryAllocation ? LDA_ENOMEM : LDA_ECUDA,
                    pre_fail_bytes ? std::string("cudaMalloc(") + std::to_string(pre_fail_bytes) +
                                         " B): " + cudaGetErrorString(copy_err)
                                   : std::string("token table copy: ") + cudaGetErrorString(copy_err));
    }
    if (pre_rows32 != H.rows32) return fail(ctx, LDA_ECUDA, "internal: θ row storage size mismatch");
    {
        // f1: with world > 1 and the recount kernel, the n_wk rows are
        // exchanged word range by word range as soon as each range is
        // recounted (overlapping the rest of the recount and the θ rebuild);
        // range p holds words [ceil(pV/P), ceil((p+1)V/P)).  Heavy-first
        // inside a range.  Results do not depend on P.
        const int64_t P = (ctx->world > 1 && !S.sweep_fused) ? std::min<int64_t>(ctx->comm_pipeline, V) : 1;
        auto range_of = [&](const lda::RecountChunk &c) {
            return static_cast<int64_t>(c.word & 0x7FFFFFFFu) * P / V;
        };
        std::stable_sort(H.rchunks.begin(), H.rchunks.end(),
                         [&](const lda::RecountChunk &a, const lda::RecountChunk &b) { return range_of(a) < range_of(b); });
        ctx->rc_begin.assign(P + 1, 0);
        ctx->w_begin.assign(P + 1, 0);
        for (int64_t p = 0; p <= P; ++p) ctx->w_begin[p] = (p * V + P - 1) / P;
        size_t i = 0;
        for (int64_t p = 0; p < P; ++p) {
            ctx->rc_begin[p] = static_cast<int64_t>(i);
            while (i < H.rchunks.size() && range_of(H.rchunks[i]) == p) ++i;
        }
        ctx->rc_begin[P] = static_cast<int64_t>(H.rchunks.size());
    }
    lda::tmark("layout done, token tables on the device");

    S.V = V;
    S.K = K;
    S.D = Dg;
    S.T = Tg;
    S.ntiles = H.ntiles;
    S.rows32 = H.rows32;
    S.alpha = ctx->alpha;
    S.beta = ctx->beta;
    S.seed = seed;

    // the small per-rank tables in one device allocation (a cudaMalloc each
    // cost ~13 ms on a fresh context: 264 ms of the load, measured)
    {
        std::vector<std::pair<void **, size_t>> parts;
        auto want = [&](auto **ptr, size_t n) {
            parts.push_back({reinterpret_cast<void **>(ptr), sizeof(**ptr) * std::max<size_t>(n, 1)});
        };
        want(&S.doc_ptr32, Dg + 1);
        want(&S.row_off32, std::max<int64_t>(Dg, 1));
        want(&S.segs, H.segs.size());
        want(&S.chunks, H.chunks.size());
        want(&S.rchunks, H.rchunks.size());
        want(&S.split_words, H.split_words.size());
        if (S.sweep_tile || S.sweep_tile_cta) {
            want(&S.titems, H.titems.size());
            want(&S.cbase, V);
        }
        want(&S.zero_words, H.zero_words.size());
        want(&S.denom, K);
        want(&S.counter, 4);
        want(&S.stat, 4);
        want(&S.ll_part, 2 * S.ll_blocks + 2);
        want(&S.ll_out, 2);
        if (!S.sweep_fused) want(&S.sweep_scratch, static_cast<size_t>(S.sweep_grid) * 2 * K);
        size_t total = 0;
        for (auto &q : parts) total += (q.second + 255) & ~size_t(255);
        char *arena = nullptr;
        DA(arena, total);
        size_t off = 0;
        for (auto &q : parts) {
            *q.first = arena + off;
            off += (q.second + 255) & ~size_t(255);
        }
    }
    S.n_chunks = static_cast<int64_t>(H.chunks.size());
    S.n_rchunks = static_cast<int64_t>(H.rchunks.size());
    S.n_split = static_cast<int64_t>(H.split_words.size());
    S.n_titems = static_cast<int64_t>(H.titems.size());
    S.n_zero_words = static_cast<int64_t>(H.zero_words.size());
    if (S.recount_gmem) {
        DA(S.recount_scratch, static_cast<size_t>(S.num_sms) * S.recount_bps * 2 * K);
        CU(cudaMemsetAsync(S.recount_scratch, 0, sizeof(int) * S.num_sms * S.recount_bps * 2 * static_cast<size_t>(K),
                           ctx->stream));
    }
    if (S.theta_gmem) {
        const size_t n = static_cast<size_t>(S.theta_grid) * (S.theta_block / 32) * (K + (K + 31) / 32);
        DA(S.theta_scratch, n);
        CU(cudaMemsetAsync(S.theta_scratch, 0, sizeof(uint32_t) * n, ctx->stream));
    }

    auto h2d = [&](void *dst, const void *src, size_t bytes) {
        return bytes ? cudaMemcpyAsync(dst, src, bytes, cudaMemcpyHostToDevice, ctx->stream) : cudaSuccess;
    };
    lda::tmark("device allocation");
    CU(h2d(S.doc_ptr32, H.doc_ptr32.data(), sizeof(uint32_t) * (Dg + 1)));
    CU(h2d(S.row_off32, H.row_off32.data(), sizeof(uint32_t) * Dg));
    CU(h2d(S.segs, H.segs.data(), sizeof(lda::Seg) * H.segs.size()));
    CU(h2d(S.chunks, H.chunks.data(), sizeof(lda::SampleChunk) * H.chunks.size()));
    CU(h2d(S.rchunks, H.rchunks.data(), sizeof(lda::RecountChunk) * H.rchunks.size()));
    CU(h2d(S.split_words, H.split_words.data(), sizeof(int32_t) * H.split_words.size()));
    CU(h2d(S.zero_words, H.zero_words.data(), sizeof(int32_t) * H.zero_words.size()));
    if (S.sweep_tile || S.sweep_tile_cta) {
        CU(h2d(S.titems, H.titems.data(), sizeof(lda::TileItem) * H.titems.size()));
        CU(h2d(S.cbase, cbase.data(), sizeof(uint64_t) * V));
    }
    CU(cudaMemsetAsync(S.rows, 0, H.rows32 * 32, ctx->stream));
    CU(cudaMemsetAsync(S.nwk, 0, (static_cast<size_t>(V) * K + K) * sizeof(int32_t), ctx->stream));

    if (dev_scatter && Tg > 0) {
        // the device layout ran on the sorter thread (joined above)
        if (sort_range) return fail(ctx, LDA_ERANGE, "too many document tiles for 32-bit layout keys");
        if (sort_err != cudaSuccess)
            return fail(ctx, sort_err == cudaErrorMemoryAllocation ? LDA_ENOMEM : LDA_ECUDA,
                        sort_where + ": " + cudaGetErrorString(sort_err));
        if (std::getenv("LDA_TIMING"))
            std::fprintf(stderr,
                         "[lda]   device layout on the sorter thread: start %.1f, scratch allocated %.1f, kernels done "
                         "%.1f, end %.1f ms\n",
                         sort_start_ms, sort_malloc_ms, sort_kernels_ms, sort_end_ms);
        lda::tmark("device layout done");
    }
    if (tile_layout) KL(lda::launch_tok_row(S, ctx->stream));
    {
        const int rs = setup_sparse_rows(ctx);
        if (rs != LDA_OK) return rs;
    }
    // a1: random init (t = 0), then the count rebuild.
    CU(cudaStreamSynchronize(ctx->stream));
    lda::tmark("H2D copies");
    KL(lda::launch_init(S, ctx->stream));
    int launches = 1;
    int r = rebuild_counts(ctx, &launches);
    if (r != LDA_OK) return r;
    CU(cudaStreamSynchronize(ctx->stream));
    lda::tmark("init + count rebuild");
    // host copies no longer needed (z moves through the device doc_map)
    H.doc_map.release();
    H.tok_row.release();
    H.tok_crank.release();
    std::vector<lda::TileItem>().swap(H.titems);
    lda::tmark("free host copies");
    ctx->loaded = true;
    ctx->sweeps = 0;
    ctx->stats.local_tokens = Tg;
    ctx->stats.local_docs = Dg;
    ctx->stats.global_tokens = ctx->T_global;
    ctx->stats.world = ctx->world;
    ctx->stats.n_sample_chunks = (S.sweep_tile || S.sweep_tile_cta) ? S.n_titems : S.n_chunks;
    ctx->stats.tile_tokens = ctx->tile_tokens_used;
    ctx->stats.n_tiles = S.ntiles;
    ctx->stats.sampler = S.sweep_tile ? 2 : (S.sweep_tile_cta ? 3 : 0);
    ctx->stats.n_sparse_words = S.sp_words;
    ctx->stats.n_stream_chunks = 1;
    ctx->stats.sum_nnz_doc = ctx->cur_nnz;
    return LDA_OK;
}

int lda_iterate(lda_ctx *ctx, int32_t n) {
    PRECHECK(ctx);
    if (!ctx->loaded) return fail(ctx, LDA_ESTATE, "no corpus loaded");
    if (n < 0) return fail(ctx, LDA_EINVAL, "negative sweep count");
    CU(cudaSetDevice(ctx->device));
    lda::DevState &S = ctx->S;
    const int per = 8;
    int r = ensure_events(ctx, static_cast<size_t>(per) * std::max(n, 1));
    if (r != LDA_OK) return r;
    while (ctx->range_ev.size() + 1 < ctx->rc_begin.size()) {
        cudaEvent_t e;
        CU(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
        ctx->range_ev.push_back(e);
    }
    const int64_t M = std::max<int64_t>(1, static_cast<int64_t>(ctx->chunks.size()));  // θ stats per sweep
    if (ctx->stat_log_cap < static_cast<size_t>(n)) {
        if (ctx->d_stat_log) {
            CU(cudaFree(ctx->d_stat_log));
            ctx->allocs.erase(std::find(ctx->allocs.begin(), ctx->allocs.end(),
                                        static_cast<void *>(ctx->d_stat_log)));
            ctx->d_stat_log = nullptr;
        }
        DA(ctx->d_stat_log, 2 * static_cast<size_t>(n) * M);
        ctx->stat_log_cap = n;
    }
    std::vector<int64_t> ll_at;  // sweeps after which the LL is logged
    int launches = 0;
    CU(cudaMemsetAsync(S.stat + 2, 0, sizeof(unsigned long long), ctx->stream));
    for (int32_t s = 0; s < n; ++s) {
        cudaEvent_t *E = ctx->ev.data() + static_cast<size_t>(per) * s;
        const uint32_t t = static_cast<uint32_t>(++ctx->sweeps);
        if (!ctx->chunks.empty()) {
            // f3: M > 1 chunks streamed through the device (WorkSchedule2)
            r = sweep_chunked(ctx, t, E, ctx->d_stat_log + 2 * static_cast<size_t>(M) * s, &launches);
            if (r != LDA_OK) return r;
            r = log_loglik(ctx, t, ll_at);
            if (r != LDA_OK) return r;
            continue;
        }
        CU(cudaEventRecord(E[0], ctx->stream));
        KL(lda::launch_sweep(S, t, ctx->stream, &launches, E[6]));
        CU(cudaEventRecord(E[1], ctx->stream));
        const int64_t P = static_cast<int64_t>(ctx->rc_begin.size()) - 1;
        if (S.sweep_fused) {
            std::swap(S.nwk, S.nwk_alt);  // the sampler wrote the next counts
        } else {
            // the ϕ update (L1273-1285), word range by word range (f1)
            for (int64_t p = 0; p < P; ++p) {
                KL(lda::launch_recount(S, ctx->stream, &launches, ctx->rc_begin[p], ctx->rc_begin[p + 1], p == 0));
                if (ctx->world > 1 && P > 1) CU(cudaEventRecord(ctx->range_ev[p], ctx->stream));
            }
        }
        CU(cudaEventRecord(E[2], ctx->stream));
        // θ update (depends only on z) on the compute stream while ϕ is
        // summed over the ranks on the comm stream (§6.2).
        // (Measured without gain: the θ rebuild on a second stream,
        // concurrent with the recount -- 7.28 + 4.32 ms overlapped vs
        // 4.98 + 2.09 ms in sequence at PubMed shape.)
        KL(lda::launch_theta(S, ctx->d_stat_log + 2 * static_cast<size_t>(s), ctx->stream, &launches));
        CU(cudaEventRecord(E[3], ctx->stream));
        if (ctx->world > 1) {
            const size_t K = static_cast<size_t>(S.K);
            if (S.sweep_fused || P == 1) {
                CU(cudaStreamWaitEvent(ctx->comm_stream, E[2], 0));
                CU(cudaEventRecord(E[7], ctx->comm_stream));
                COMM(allreduce_i32(S.nwk, static_cast<size_t>(S.V) * K + K, ctx->comm_stream, e_));
            } else {
                for (int64_t p = 0; p < P; ++p) {
                    // rows of range p; the last range carries n_k (complete after every range's recount)
                    const size_t r0 = static_cast<size_t>(ctx->w_begin[p]) * K;
                    const size_t r1 = static_cast<size_t>(ctx->w_begin[p + 1]) * K + (p == P - 1 ? K : 0);
                    CU(cudaStreamWaitEvent(ctx->comm_stream, ctx->range_ev[p], 0));
                    if (p == 0) CU(cudaEventRecord(E[7], ctx->comm_stream));
                    if (r1 > r0) COMM(allreduce_i32(S.nwk + r0, r1 - r0, ctx->comm_stream, e_));
                }
            }
            CU(cudaEventRecord(E[4], ctx->comm_stream));
            CU(cudaStreamWaitEvent(ctx->stream, E[4], 0));
        }
        CU(cudaEventRecord(E[5], ctx->stream));
        r = log_loglik(ctx, t, ll_at);
        if (r != LDA_OK) return r;
    }
    CU(cudaStreamSynchronize(ctx->stream));
    if (ctx->h2d_stream) CU(cudaStreamSynchronize(ctx->h2d_stream));
    if (ctx->d2h_stream) CU(cudaStreamSynchronize(ctx->d2h_stream));
    ctx->ll_sweep = ll_at;
    ctx->ll_value.assign(ll_at.size(), 0.0);
    for (size_t i = 0; i < ll_at.size(); ++i)
        ctx->ll_value[i] = ctx->ll_pending[i] / static_cast<double>(ctx->T_global > 0 ? ctx->T_global : 1);
    ctx->ll_pending.clear();
    unsigned long long n_exact = 0;
    CU(cudaMemcpy(&n_exact, S.stat + 2, sizeof(n_exact), cudaMemcpyDeviceToHost));
    ctx->stats.n_exact_redraws = static_cast<int64_t>(n_exact);
    std::vector<unsigned long long> hs(2 * static_cast<size_t>(n));
    if (n) {
        std::vector<unsigned long long> hm(2 * static_cast<size_t>(n) * M);
        CU(cudaMemcpy(hm.data(), ctx->d_stat_log, hm.size() * sizeof(unsigned long long), cudaMemcpyDeviceToHost));
        for (size_t i = 0; i < static_cast<size_t>(n); ++i)
            for (int64_t m = 0; m < M; ++m) {
                hs[2 * i] += hm[2 * (i * M + m)];
                hs[2 * i + 1] += hm[2 * (i * M + m) + 1];
            }
    }
    lda_stats &st = ctx->stats;
    st.last_n = n;
    st.sweeps_done = static_cast<int64_t>(ctx->sweeps);
    st.ms_total = st.ms_sample = st.ms_recount = st.ms_theta = st.ms_allreduce = st.ms_table = 0;
    st.ms_allreduce_exposed = 0;
    st.ms_last_sweep = st.ms_last_sample = 0;
    ctx->log_ms.assign(n, 0);
    ctx->log_ms_sample.assign(n, 0);
    ctx->log_ms_recount.assign(n, 0);
    ctx->log_ms_theta.assign(n, 0);
    ctx->log_ms_comm.assign(n, 0);
    ctx->log_nnz_tok.assign(n, 0);
    ctx->log_nnz_doc.assign(n, 0);
    for (int32_t s = 0; s < n; ++s) {
        cudaEvent_t *E = ctx->ev.data() + static_cast<size_t>(per) * s;
        float a = 0, b = 0, c = 0, d = 0, tot = 0;
        CU(cudaEventElapsedTime(&a, E[0], E[1]));
        float tb = 0;
        CU(cudaEventElapsedTime(&tb, E[0], E[6]));
        st.ms_table += tb;
        CU(cudaEventElapsedTime(&b, E[1], E[2]));
        CU(cudaEventElapsedTime(&c, E[2], E[3]));
        CU(cudaEventElapsedTime(&tot, E[0], E[5]));
        float x = 0;
        if (ctx->world > 1) {
            // raw exchange time: from the first range's start to the end (includes waits for later ranges)
            CU(cudaEventElapsedTime(&d, E[7], E[4]));
            // exposed: the compute stream's wait for the allreduce after the θ rebuild
            CU(cudaEventElapsedTime(&x, E[3], E[5]));
        }
        st.ms_allreduce_exposed += x;
        st.ms_sample += a;
        st.ms_recount += b;
        st.ms_theta += c;
        st.ms_allreduce += d;
        st.ms_total += tot;
        ctx->log_ms[s] = tot;
        ctx->log_ms_sample[s] = a;
        ctx->log_ms_recount[s] = b;
        ctx->log_ms_theta[s] = c;
        ctx->log_ms_comm[s] = d;
        // sweep s sampled against the θ built before it
        ctx->log_nnz_tok[s] = ctx->cur_lnnz;
        ctx->cur_lnnz = static_cast<int64_t>(hs[2 * s]);
        ctx->cur_nnz = static_cast<int64_t>(hs[2 * s + 1]);
        ctx->log_nnz_doc[s] = ctx->cur_nnz;
        if (s == n - 1) {
            st.ms_last_sweep = tot;
            st.ms_last_sample = a;
            st.sum_nnz_tok = ctx->log_nnz_tok[s];
        }
    }
    st.sum_nnz_doc = ctx->cur_nnz;
    st.n_launches = launches;
    // SURVEY §8(d) byte model of the last sweep (this rank): B_alg and the
    // sampling kernel's share B_sample
    if (n > 0) {
        const double Tg = static_cast<double>(S.T), VK = static_cast<double>(S.V) * S.K;
        const double ntok = static_cast<double>(st.sum_nnz_tok);
        st.bytes_alg = 20.0 * Tg + 4.0 * ntok + 8.0 * VK + 4.0 * static_cast<double>(st.sum_nnz_doc) +
                       8.0 * static_cast<double>(S.D);
        st.bytes_sample = 14.0 * Tg + 4.0 * ntok + 4.0 * VK;
    }
    return LDA_OK;
}

int lda_get_loglik_log(lda_ctx *ctx, int32_t cap, int64_t *sweep, double *ll_per_token, int32_t *n_out) {
    PRECHECK(ctx);
    const int32_t n = static_cast<int32_t>(ctx->ll_sweep.size());
    if (n_out) *n_out = n;
    const int32_t m = std::min(n, std::max(cap, 0));
    for (int32_t i = 0; i < m; ++i) {
        if (sweep) sweep[i] = ctx->ll_sweep[i];
        if (ll_per_token) ll_per_token[i] = ctx->ll_value[i];
    }
    return LDA_OK;
}

int lda_get_sweep_log(lda_ctx *ctx, int32_t cap, double *ms_sweep, double *ms_sample, double *ms_recount,
                      double *ms_theta, double *ms_allreduce, int64_t *sum_nnz_tok, int64_t *sum_nnz_doc,
                      int32_t *n_out) {
    PRECHECK(ctx);
    const int32_t n = static_cast<int32_t>(ctx->log_ms.size());
    if (n_out) *n_out = n;
    const int32_t m = std::min(n, std::max(cap, 0));
    for (int32_t s = 0; s < m; ++s) {
        if (ms_sweep) ms_sweep[s] = ctx->log_ms[s];
        if (ms_sample) ms_sample[s] = ctx->log_ms_sample[s];
        if (ms_recount) ms_recount[s] = ctx->log_ms_recount[s];
        if (ms_theta) ms_theta[s] = ctx->log_ms_theta[s];
        if (ms_allreduce) ms_allreduce[s] = ctx->log_ms_comm[s];
        if (sum_nnz_tok) sum_nnz_tok[s] = ctx->log_nnz_tok[s];
        if (sum_nnz_doc) sum_nnz_doc[s] = ctx->log_nnz_doc[s];
    }
    return LDA_OK;
}

int lda_loglik(lda_ctx *ctx, double *ll) {
    PRECHECK(ctx);
    if (!ll) return fail(ctx, LDA_EINVAL, "null output");
    if (!ctx->loaded) return fail(ctx, LDA_ESTATE, "no corpus loaded");
    CU(cudaSetDevice(ctx->device));
    double h[2];
    int r = loglik_pair(ctx, h);
    if (r != LDA_OK) return r;
    *ll = (h[0] + h[1]) / static_cast<double>(ctx->T_global > 0 ? ctx->T_global : 1);
    return LDA_OK;
}

int lda_get_counts(lda_ctx *ctx, int32_t *n_wk, int32_t *n_k, int64_t *ndk_ptr, uint16_t *ndk_topic,
                   int32_t *ndk_count, int64_t ndk_capacity, int64_t *ndk_nnz_out, uint16_t *z) {
    PRECHECK(ctx);
    if (!ctx->loaded) return fail(ctx, LDA_ESTATE, "no corpus loaded");
    CU(cudaSetDevice(ctx->device));
    CU(cudaStreamSynchronize(ctx->stream));
    const lda::DevState &S = ctx->S;
    const lda::HostLayout &H = ctx->H;
    if (n_wk) CU(cudaMemcpy(n_wk, S.nwk, sizeof(int32_t) * S.V * S.K, cudaMemcpyDeviceToHost));
    if (n_k) CU(cudaMemcpy(n_k, S.nwk + static_cast<size_t>(S.V) * S.K, sizeof(int32_t) * S.K,
                           cudaMemcpyDeviceToHost));
    if (ndk_ptr || ndk_topic || ndk_count || ndk_nnz_out) {
        // θ rows: the device copy, or (M > 1 chunks) the chunks' host copies
        struct Src {
            const uint32_t *rows;
            const std::vector<uint32_t> *off;
            int64_t D;
        };
        std::vector<Src> src;
        std::vector<uint32_t> rows;
        if (ctx->chunks.empty()) {
            rows.resize(H.rows32 * 8);
            CU(cudaMemcpy(rows.data(), S.rows, rows.size() * sizeof(uint32_t), cudaMemcpyDeviceToHost));
            src.push_back({rows.data(), &H.row_off32, S.D});
        } else {
            if (ctx->d2h_stream) CU(cudaStreamSynchronize(ctx->d2h_stream));
            for (auto &c : ctx->chunks) src.push_back({c->hrows, &c->H.row_off32, c->D});
        }
        int64_t nnz = 0;
        for (const Src &q : src)
            for (int64_t d = 0; d < q.D; ++d) nnz += q.rows[static_cast<size_t>((*q.off)[d]) * 8];
        if (ndk_nnz_out) *ndk_nnz_out = nnz;
        if ((ndk_topic || ndk_count) && ndk_capacity < nnz)
            return fail(ctx, LDA_ERANGE, "ndk_capacity smaller than nnz");
        int64_t pos = 0, dg = 0;
        for (const Src &q : src)
            for (int64_t d = 0; d < q.D; ++d, ++dg) {
                const uint32_t *row = q.rows + static_cast<size_t>((*q.off)[d]) * 8;
                if (ndk_ptr) ndk_ptr[dg] = pos;
                for (uint32_t j = 0; j < row[0]; ++j, ++pos) {
                    if (ndk_topic) ndk_topic[pos] = static_cast<uint16_t>(row[1 + j] >> (S.K > 16384 ? 16 : 18));
                    if (ndk_count) ndk_count[pos] = static_cast<int32_t>(row[1 + j] & 0xFFFFu);
                }
            }
        if (ndk_ptr) ndk_ptr[dg] = pos;
    }
    if (z && S.T && !ctx->chunks.empty()) {
        // M > 1: the chunks' word-major host copies, into document order
        if (ctx->d2h_stream) CU(cudaStreamSynchronize(ctx->d2h_stream));
        for (auto &c : ctx->chunks)
            for (int64_t i = 0; i < c->T; ++i) z[c->tok_begin + i] = c->hz[c->H.doc_map[i]];
        return LDA_OK;
    }
    if (z && S.T) {
        // z into document order on the device (the θ rebuild's gather), then D2H
        uint16_t *zd = S.z_doc;
        if (!zd) CU(cudaMalloc(&zd, sizeof(uint16_t) * (S.T + 8)));
        int r = lda::launch_gather_z(S, zd, ctx->stream);
        cudaError_t ce = r == cudaSuccess ? cudaMemcpyAsync(z, zd, sizeof(uint16_t) * S.T, cudaMemcpyDeviceToHost,
                                                            ctx->stream)
                                          : static_cast<cudaError_t>(r);
        if (ce == cudaSuccess) ce = cudaStreamSynchronize(ctx->stream);
        if (zd != S.z_doc) cudaFree(zd);
        if (ce != cudaSuccess) return fail(ctx, LDA_ECUDA, std::string("z gather: ") + cudaGetErrorString(ce));
    }
    return LDA_OK;
}

int lda_set_z(lda_ctx *ctx, const uint16_t *z) {
    PRECHECK(ctx);
    if (!ctx->loaded) return fail(ctx, LDA_ESTATE, "no corpus loaded");
    const lda::DevState &S = ctx->S;
    if (!z && S.T) return fail(ctx, LDA_EINVAL, "null z");
    for (int64_t i = 0; i < S.T; ++i)
        if (z[i] >= S.K) return fail(ctx, LDA_EINVAL, "topic id >= K");
    CU(cudaSetDevice(ctx->device));
    if (!ctx->chunks.empty()) {
        // M > 1: into the chunks' word-major host copies, then the rebuild
        CU(cudaStreamSynchronize(ctx->d2h_stream));
        for (auto &c : ctx->chunks)
            for (int64_t i = 0; i < c->T; ++i) c->hz[c->H.doc_map[i]] = z[c->tok_begin + i];
        int launches = 0;
        return chunked_rebuild(ctx, false, &launches);
    }
    if (S.T) {
        // H2D in document order, scattered to word-major positions on the device
        uint16_t *zd = nullptr;
        CU(cudaMalloc(&zd, sizeof(uint16_t) * S.T));
        cudaError_t ce = cudaMemcpyAsync(zd, z, sizeof(uint16_t) * S.T, cudaMemcpyHostToDevice, ctx->stream);
        if (ce == cudaSuccess) ce = static_cast<cudaError_t>(lda::launch_scatter_z(S, zd, ctx->stream));
        if (ce == cudaSuccess) ce = cudaStreamSynchronize(ctx->stream);
        cudaFree(zd);
        if (ce != cudaSuccess) return fail(ctx, LDA_ECUDA, std::string("z scatter: ") + cudaGetErrorString(ce));
    }
    int launches = 0;
    int r = rebuild_counts(ctx, &launches);
    if (r != LDA_OK) return r;
    CU(cudaStreamSynchronize(ctx->stream));
    return LDA_OK;
}

int lda_get_stats(lda_ctx *ctx, lda_stats *out) {
    PRECHECK(ctx);
    if (!out) return fail(ctx, LDA_EINVAL, "null output");
    *out = ctx->stats;
    return LDA_OK;
}

int lda_get_stream(lda_ctx *ctx, void **stream) {
    PRECHECK(ctx);
    if (!stream) return fail(ctx, LDA_EINVAL, "null output");
    if (!ctx->loaded) return fail(ctx, LDA_ESTATE, "no corpus loaded");
    *stream = ctx->stream;
    return LDA_OK;
}

void lda_destroy(lda_ctx *ctx) {
    if (!ctx) return;
    if (ctx->stream || !ctx->allocs.empty()) {
        cudaSetDevice(ctx->device);
        if (ctx->stream) cudaStreamSynchronize(ctx->stream);
        for (cudaStream_t st : {ctx->h2d_stream, ctx->d2h_stream})
            if (st) {
                cudaStreamSynchronize(st);
                cudaStreamDestroy(st);
            }
        for (auto &b : ctx->slot)
            for (cudaEvent_t e : {b.in, b.done, b.free_})
                if (e) cudaEventDestroy(e);
        for (auto &c : ctx->chunks) {
            if (c->registered) {
                cudaHostUnregister(c->H.tok_row.data());
                cudaHostUnregister(c->H.doc_map.data());
            }
            if (c->hz) cudaFreeHost(c->hz);
            if (c->hrows) cudaFreeHost(c->hrows);
        }
        ctx->chunks.clear();
        for (void *p : ctx->allocs) cudaFree(p);
        for (cudaEvent_t e : ctx->ev) cudaEventDestroy(e);
        for (cudaEvent_t e : ctx->range_ev) cudaEventDestroy(e);
        if (ctx->stream) cudaStreamDestroy(ctx->stream);
        if (ctx->comm_stream) cudaStreamDestroy(ctx->comm_stream);
    }
    ctx->comm.reset();
    delete ctx;
}

}  // extern "C"

int lda_layout_selfcheck(int64_t D, int32_t V, int32_t K, const int64_t *doc_ptr, const int32_t *words,
                         int32_t sampler, int64_t tile_tokens, int64_t chunk_tokens, int64_t tail_per_tile,
                         int64_t *out_stats, char *msg, int32_t msg_cap) {
    auto bad = [&](const std::string &m) {
        if (msg && msg_cap > 0) {
            std::strncpy(msg, m.c_str(), static_cast<size_t>(msg_cap) - 1);
            msg[msg_cap - 1] = 0;
        }
        return static_cast<int>(LDA_EINVAL);
    };
    if (D < 0 || V < 1 || K < 1 || !doc_ptr || sampler < 0 || sampler > 3 || sampler == 1 || chunk_tokens < 1)
        return bad("invalid arguments");
    bool range_err = false;
    std::string v = lda::validate_corpus(doc_ptr, words, D, V, &range_err, nullptr, 0);
    if (!v.empty()) return bad(v);
    const int64_t T = doc_ptr[D];
    std::vector<int64_t> cbase(V, 0), wc(V, 0);
    lda::word_histogram(words, T, V, 0, wc.data());
    lda_canonical_bases(V, 1, 0, wc.data(), cbase.data(), nullptr);
    lda::HostLayout H;
    const int layout = sampler >= 2 ? 2 : sampler;
    std::string e = lda::build_layout(doc_ptr, words, D, V, K, cbase.data(), tile_tokens, chunk_tokens, 65536, 0,
                                      layout, tail_per_tile, H);
    if (!e.empty()) return bad(e);
    // doc_map: a permutation; tok_row: the row of the token's document
    std::vector<int64_t> word_at(T, -1), tokidx_at(T, -1);
    for (int64_t d = 0; d < D; ++d)
        for (int64_t i = doc_ptr[d]; i < doc_ptr[d + 1]; ++i) {
            const uint32_t p = H.doc_map[i];
            if (p >= static_cast<uint64_t>(T)) return bad("doc_map out of range");
            if (word_at[p] >= 0) return bad("doc_map is not a permutation");
            word_at[p] = words[i];
            tokidx_at[p] = i;
            if (H.tok_row[p] != H.row_off32[d]) return bad("tok_row is not the row of the token's document");
        }
    // canonical rank of each token by brute force: order within its word in (d, j) order
    std::vector<int64_t> seen(V, 0), crank_at(T, -1);
    for (int64_t i = 0; i < T; ++i) crank_at[H.doc_map[i]] = seen[words[i]]++;
    // runs: each word's runs (segs) cover exactly its tokens and hold only that word
    int64_t runs = 0;
    {
        // per word: runs {pos, vstart} ..., then a sentinel {0, n_w}
        size_t sidx = 0;
        for (int32_t w = 0; w < V; ++w) {
            int64_t covered = 0;
            while (sidx + 1 < H.segs.size() && H.segs[sidx].vstart < static_cast<uint64_t>(wc[w])) {
                const lda::Seg &sg = H.segs[sidx];
                const uint32_t len = H.segs[sidx + 1].vstart - sg.vstart;
                for (uint32_t j = 0; j < len; ++j)
                    if (word_at[static_cast<size_t>(sg.pos) + j] != w) return bad("a word's run holds another word");
                covered += len;
                ++runs;
                ++sidx;
            }
            if (sidx >= H.segs.size() || H.segs[sidx].vstart != static_cast<uint64_t>(wc[w]))
                return bad("missing run sentinel");
            ++sidx;
            if (covered != wc[w]) return bad("a word's runs do not cover its tokens");
        }
    }
    // tile-sampler items: canonical ranks crank0 + j, every token once
    if (layout == 2) {
        std::vector<uint8_t> hit(T, 0);
        for (const lda::TileItem &it : H.titems) {
            for (uint32_t j = 0; j < it.n; ++j) {
                const uint64_t p = static_cast<uint64_t>(it.pos) + j;
                if (p >= static_cast<uint64_t>(T)) return bad("item out of range");
                if (hit[p]) return bad("a token is in two items");
                hit[p] = 1;
                if (word_at[p] != static_cast<int64_t>(it.word)) return bad("an item holds another word");
                if (crank_at[p] != static_cast<int64_t>(it.crank0) + j)
                    return bad("item canonical rank crank0 + j differs from the brute-force rank");
            }
        }
        for (int64_t p = 0; p < T; ++p)
            if (!hit[p]) return bad("a token is in no item");
    } else {
        for (int64_t p = 0; p < T; ++p)
            if (static_cast<int64_t>(H.tok_crank[p]) != crank_at[p]) return bad("tok_crank differs from the brute-force rank");
    }
    int64_t ntail = 0;
    if (layout == 2 && H.ntiles > 1) {
        // tail words: exactly one run, in the last tile
        for (int32_t w = 0; w < V; ++w)
            if (wc[w] > 0 && wc[w] < tail_per_tile * (H.ntiles - 1)) ++ntail;
    }
    if (out_stats) {
        out_stats[0] = H.ntiles;
        out_stats[1] = static_cast<int64_t>(layout == 2 ? H.titems.size() : H.chunks.size());
        out_stats[2] = ntail;
        out_stats[3] = runs;
    }
    return LDA_OK;
}
