/*
 * include/lda.h — C ABI of the B200-native LDA collapsed-Gibbs sweep
 * (the hot path of CuLDA_CGS, Xie, Liang, Li, Tan, HPDC'19).
 *
 * Citations "L<n>" are lines of the paper transcript /root/reference/PAPER.md;
 * "X<n>" are the readings of ambiguous passages listed in DESIGN.md.
 *
 * What the library computes (§2.1, §6):
 *   corpus: D documents of tokens, each token an instance of a word in [0,V)
 *           (L369-383).
 *   model : θ (n_dk, doc-topic counts, sparse), ϕ (n_wk, word-topic counts,
 *           dense) and n_k = Σ_w n_wk (L391-397, Eq. 1 denominator L407).
 *   sweep : every token draws a new topic from
 *             p(k) ∝ (n_dk + α)(n_wk + β) / (n_k + Vβ)            (Eq. 1)
 *           against the counts frozen at the start of the sweep (L415-421,
 *           X3), via the split p = p1 + p2 (Eq. 6-8),
 *           one Philox4x32-10 uniform per token keyed by (seed; canonical
 *           token index c, sweep t) (X9); then n_wk, n_k and θ are rebuilt
 *           (§6.2).  Multi-GPU: documents are partitioned, n_wk/n_k
 *           are sum-allreduced after every sweep (Eq. 4).
 *
 * Conventions for every call:
 *   - Return 0 (LDA_OK) or a negative lda_status.  No exceptions cross the ABI.
 *   - Input pointers are HOST pointers, borrowed for the duration of the call
 *     only (the library copies).  Output buffers are caller-allocated host
 *     memory; passing NULL skips that output.
 *   - A context is single-threaded: do not call into one context from two
 *     threads at once.
 *   - Sticky failures: a CUDA or NCCL error marks the context failed; every
 *     later call on it returns the same code until lda_destroy.
 *     lda_last_error() gives a human-readable detail.
 *   - Call order: lda_create -> [lda_set_option]* -> [lda_init_dist] ->
 *     lda_load_corpus -> (lda_iterate | lda_loglik | lda_get_counts |
 *     lda_get_stats | lda_set_z)* -> lda_destroy.  Calls that need a corpus
 *     return LDA_ESTATE before a successful lda_load_corpus.
 */
#ifndef LDA_H
#define LDA_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct lda_ctx lda_ctx; /* opaque; owned by the library */

typedef enum {
    LDA_OK = 0,
    LDA_EINVAL = -1, /* invalid argument or corpus */
    LDA_ERANGE = -2, /* a size exceeds a representable range / buffer too small */
    LDA_ENOMEM = -3, /* host or device allocation failed */
    LDA_ECUDA = -4,  /* CUDA runtime error (including: no device) */
    LDA_ENCCL = -5,  /* NCCL error */
    LDA_ESTATE = -6  /* call out of order */
} lda_status;

/* Per-call statistics of the last lda_iterate (device time from CUDA events
 * on the library's streams). */
typedef struct lda_stats {
    int64_t sweeps_done;    /* global sweep counter t after the last call */
    int64_t local_tokens;   /* T_g: tokens held by this rank */
    int64_t local_docs;     /* D_g */
    int64_t global_tokens;  /* T */
    int32_t last_n;         /* sweeps in the last lda_iterate call */
    int32_t world;          /* ranks */
    double ms_total;        /* compute-stream time of the last call, all sweeps */
    double ms_sample;       /* prologue + sampling kernel (Alg. 2, K1) */
    double ms_recount;      /* n_wk / n_k rebuild (K2) */
    double ms_theta;        /* θ rebuild (K3+K4) */
    double ms_allreduce;    /* raw allreduce time on the comm stream (0 if world==1) */
    double ms_last_sweep;   /* compute-stream time of the last sweep only */
    double ms_last_sample;  /* sampling kernel time of the last sweep only */
    int64_t sum_nnz_tok;    /* Σ_t nnz_{d(t)} read by the last sweep's sampler */
    int64_t sum_nnz_doc;    /* Σ_d nnz_d of θ after the last sweep */
    int64_t n_launches;     /* library kernels launched by the last call */
    int64_t n_sample_chunks;/* sampler work items (word chunks) */
    int64_t n_exact_redraws;/* samplers 2, 3: tokens of the last lda_iterate
                               call whose fp32 draw could not be certified and
                               that were redrawn by the exact fp64 walk */
    double ms_table;        /* samplers 2, 3: the per-word table kernel (a3), part of
                               ms_sample; ms_sample - ms_table = sampling kernel */
    double ms_allreduce_exposed; /* world > 1: time the compute stream waited for
                               the allreduce after the θ rebuild (the part of
                               ms_allreduce not hidden behind it) */
    int64_t tile_tokens;    /* document tile size the layout used (0: one tile) */
    int32_t n_tiles;        /* tiles, including the tail tile */
    int32_t sampler;        /* the sampler that runs: 0, 2 or 3 (see "sampler") */
    double bytes_alg;       /* SURVEY §8(d) algorithmic bytes of the last sweep on
                               this rank: 20·T_g + 4·Σ_t nnz_d(t) + 8·V·K
                               + 4·Σ_d nnz'_d + 8·D_g */
    double bytes_sample;    /* the sampling kernel's share of it:
                               14·T_g + 4·Σ_t nnz_d(t) + 4·V·K */
    int64_t n_stream_chunks;/* M: chunks streamed per sweep (option stream_chunks;
                               1 = the corpus stays resident, WorkSchedule1) */
    int64_t n_sparse_words; /* sampler 3 (K > 4096): words whose tables are
                               built from sparse rows (option "sparse_words") */
} lda_stats;

/* Create a context.  D = global number of documents, V = vocabulary size,
 * K = number of topics, α, β = Dirichlet hyper-parameters (Eq. 1; the paper
 * uses α = 50/K, β = 0.01 at L1339, X1).  No device work is done.
 * Errors: LDA_EINVAL unless D >= 1, V >= 1, 1 <= K <= 65536 (topic ids are
 * uint16, L1239-1243), α and β finite and > 0.  For K > 16384 θ entries are
 * packed topic << 16 | count, the K-length histograms of the recount and the
 * θ rebuild live in global scratch, and the sampler is the lane-per-token
 * one (sampler 0).  *out is set to NULL on error. */
int lda_create(int64_t D, int32_t V, int32_t K, double alpha, double beta, lda_ctx **out);

/* Set an integer option before lda_load_corpus (LDA_ESTATE after).  Keys:
 *   "device"        CUDA device ordinal (default 0)
 *   "exclude_self"  0 (default; Eq. 1 as printed, X2) or 1 (remove the
 *                   token's own old topic from the counts it draws against;
 *                   runs on sampler 0)
 *   "tile_tokens"   -1 (default, auto): split the documents into tiles whose
 *                   θ rows fill about half the L2 (one tile if all rows fit)
 *                   and sample tile by tile, so that every tile's rows are
 *                   read from HBM about once per sweep; 0: one tile; n > 0:
 *                   tiles of about n tokens
 *   "chunk_tokens"  max tokens per sampling work item (default 4096)
 *   "recount_tokens" max tokens per n_wk recount work item (default 65536)
 *   "threads"       host threads for corpus preparation (default: all)
 *   "sampler"       -1 (default): 2 if K <= 4096, else 3.
 *                   2: tile sampler -- work items are the tokens of one word
 *                   inside one document tile, queued tile by tile so the
 *                   tiles' θ rows stay in L2; one warp per item, the word's
 *                   p* and dense-prefix table (built once per sweep)
 *                   bulk-copied to shared memory, four lanes walk a θ row
 *                   line by line, draws in fp32 certified against rigorous
 *                   error bounds (uncertain tokens redrawn in fp64).
 *                   3: the tile sampler with the word tables shared by the
 *                   warps of a CTA (several buffers in flight) -- large K;
 *                   same draws as 2.
 *                   0: lane-per-token fp64 sampler (32-byte row blocks); the
 *                   path of exclude_self = 1.
 *                   2 and 3 fall back to 0 with exclude_self = 1 or when
 *                   their shared-memory layout does not fit.  The samplers
 *                   differ only in rounding at a CDF boundary (draws differ
 *                   only within fp64 rounding of it).
 *   "tail_per_tile" samplers 2, 3: words with fewer than this many tokens
 *                   per document tile on average are sampled as one
 *                   corpus-wide item each (default 48; 0 = off).  Sampler 3
 *                   scales it by K/1024 (its per-item table copy grows
 *                   with K).
 *   "fused_recount" samplers 2, 3: 0 (default) = n_wk / n_k rebuilt after
 *                   the sampler by the segmented recount kernel (per-word
 *                   shared histograms over the word's runs, no global atomics
 *                   except for words split over recount chunks; measured
 *                   2.7 % faster per sweep at PubMed shape); 1 = accumulated
 *                   by the sampler itself (warp-aggregated reductions).  Same
 *                   counts.
 *   "stream_chunks" M >= 1 (default 1).  M > 1: out-of-HBM streaming (Alg. 1
 *                   WorkSchedule2, L835-859, §5.1): the rank's
 *                   documents are cut into M token-balanced chunks whose
 *                   token tables, z and θ rows stay in page-locked host
 *                   memory; every sweep streams each chunk through one of two
 *                   device slots (the transfer of chunk m+1 overlaps the
 *                   sampling of chunk m, L925-931), n_wk and the word tables
 *                   stay resident.  Needs sampler 2 or 3 (exclude_self = 0).
 *                   Same draws as M = 1.  With M > 1 ms_sample holds the
 *                   whole chunk loop (recount and θ inside it).
 *   "sparse_words"  sampler 3 at K > 4096 with K % 4 == 0 (f2; SparseLDA's
 *                   split p*(k) = β/(n_k+Vβ) + n_wk/(n_k+Vβ), ref [32], L999):
 *                   words with at most this many tokens in the corpus get no
 *                   O(K) p* row in their table; the table kernel writes their
 *                   nonzero topics instead and the sampler rebuilds the row in
 *                   shared memory from the smoothing row β/(n_k+Vβ), shared by
 *                   all words, patched at those topics.  -1: K/4; 0
 *                   (default): off -- measured slower on B200 at NYTimes
 *                   shape, K = 8192 (19.90 vs 19.45 ms per sweep: the table
 *                   kernel is latency-bound, not write-bound, and the bulk
 *                   copy of a dense row costs the sampler's warps nothing
 *                   while the patching does).  Same draws (the tables are
 *                   bit-identical).
 *   "comm_pipeline" world > 1 with the recount kernel (fused_recount = 0):
 *                   recount n_wk in this many word ranges (default 4) and
 *                   start the exchange (Eq. 4) of each range's rows as soon
 *                   as it is recounted, overlapping the rest of the recount
 *                   and the θ rebuild (§6.2).  Same counts.
 *   "certify_slack" samplers 2, 3, tests only: multiply every certification
 *                   bound by this factor (default 1) -- more tokens take the
 *                   exact fp64 redraw; the draws must not change
 *   "loglik_every"  n > 0: lda_iterate evaluates the LL/token (as lda_loglik)
 *                   after every sweep t with t % n == 0, outside the sweep's
 *                   timed phases; read with lda_get_loglik_log (default 0)
 * Results do not depend on chunk_tokens, recount_tokens, tile_tokens or
 * threads (the draw of every token is a function of the frozen counts and
 * its canonical index only).
 * Unknown key or bad value: LDA_EINVAL. */
int lda_set_option(lda_ctx *ctx, const char *key, int64_t value);

/* Multi-GPU: join a communicator of `world` ranks as `rank` (one process per
 * GPU).  nccl_unique_id points to the 128-byte ncclUniqueId that rank 0 made
 * with lda_nccl_unique_id and the caller broadcast (e.g. through
 * torch.distributed).  Must precede lda_load_corpus.  world == 1 is allowed
 * (no communicator is made).  Errors: LDA_EINVAL, LDA_ESTATE, LDA_ENCCL. */
int lda_init_dist(lda_ctx *ctx, int32_t rank, int32_t world, const void *nccl_unique_id);

/* Write a fresh 128-byte ncclUniqueId to out128 (host-only helper). */
int lda_nccl_unique_id(void *out128);

/* In-process multi-GPU: a group of `world` ranks (1..16) in ONE process,
 * each rank a context driven by its own host thread, on its own GPU (P2P
 * over NVLink) or several on one GPU.  The n_wk/n_k exchange of Eq. 4
 * (L935-937) reads the peers' device buffers directly: a reduce-scatter
 * kernel (rank r sums slice r over all ranks in place), then an all-gather
 * kernel, ordered by host barriers.  Collective calls (lda_load_corpus,
 * lda_iterate, lda_loglik, lda_set_z) must be made by every rank's thread
 * concurrently; a rank that fails or does not arrive within 600 s breaks
 * the group (every later collective fails with LDA_ECUDA).
 * lda_peer_group_create: *out receives the group handle (LDA_EINVAL for a
 * bad world).  lda_init_peer: join as `rank` before lda_load_corpus
 * (LDA_EINVAL: bad or duplicate rank; LDA_ESTATE: after load or after
 * lda_init_dist).  The group's state is shared by its contexts:
 * lda_peer_group_destroy may be called once every rank has joined. */
typedef struct lda_peer_group lda_peer_group;
int lda_peer_group_create(int32_t world, lda_peer_group **out);
int lda_init_peer(lda_ctx *ctx, lda_peer_group *group, int32_t rank);
void lda_peer_group_destroy(lda_peer_group *group);

/* Token-balanced contiguous document partition (§4 "evenly
 * partitioned by number of tokens", X21): rank g owns documents
 * [doc_begin[g], doc_begin[g+1]), where doc_begin[g] is the first d with
 * doc_ptr[d] >= ceil(g*T/world), doc_begin[0] = 0, doc_begin[world] = D.
 * doc_ptr: D+1 non-decreasing offsets (doc_ptr[0] == 0, T = doc_ptr[D]);
 * doc_begin: world+1 outputs.  Host-only.  Errors: LDA_EINVAL. */
int lda_partition_docs(int64_t D, const int64_t *doc_ptr, int32_t world, int64_t *doc_begin);

/* Canonical-index bases for a rank (host-only; lda_load_corpus uses it).
 * The canonical index of a token is its position in the stable sort of the
 * whole corpus by (word, document, position) (X18; the paper's word-first
 * order, L1189-1191).  With documents partitioned into contiguous rank
 * ranges, rank g's tokens of word w are one contiguous run of that order,
 * starting at cbase[w] = Σ_{w'<w} T(w') + Σ_{g'<g} T_{g'}(w).
 *   word_counts: world*V per-rank word histograms, rank-major
 *   cbase: V outputs; total (may be NULL): T = Σ of all counts. */
int lda_canonical_bases(int32_t V, int32_t world, int32_t rank, const int64_t *word_counts, int64_t *cbase,
                        int64_t *total);

/* Host-only diagnostic (no device needed): build the token layout that
 * lda_load_corpus would build for a one-rank corpus (doc_ptr: D+1 offsets,
 * words: T ids < V) with the given sampler (0, 2 or 3), tile_tokens,
 * chunk_tokens and tail_per_tile, and check its invariants against brute
 * force: doc_map is a permutation of [0, T); tok_row[doc_map[i]] is the θ
 * row of token i's document; every (tile, word) run holds only that word;
 * the runs of a word cover exactly its tokens; for the tile samplers every
 * work item's token pos + j has canonical rank crank0 + j (the rank of the
 * token within its word in (document, position) order, X18) and the items
 * cover every token once.  out_stats (may be NULL) receives {tiles, items,
 * tail words, runs}.  Returns LDA_OK, or LDA_EINVAL with a message in
 * msg (msg_cap bytes) when an invariant fails or the input is invalid. */
int lda_layout_selfcheck(int64_t D, int32_t V, int32_t K, const int64_t *doc_ptr, const int32_t *words,
                         int32_t sampler, int64_t tile_tokens, int64_t chunk_tokens, int64_t tail_per_tile,
                         int64_t *out_stats, char *msg, int32_t msg_cap);

/* Diagnostic (tests): the library's device radix sort -- a stable LSD sort
 * of n (key, value) pairs by the low `bits` bits of the keys (8 bits per
 * pass; lda_load_corpus uses it to build the tile layout's doc-word map on
 * the device).  Host arrays in, host arrays out; device scratch is
 * allocated and freed by the call.  Returns 0, LDA_EINVAL or LDA_ECUDA. */
int lda_debug_radix_sort(const uint32_t *keys, const uint32_t *vals, int64_t n, int32_t bits, uint32_t *out_keys,
                         uint32_t *out_vals);

/* Diagnostic (tests): the NCCL backend of the exchange end to end with one
 * rank on `device` (this environment has one GPU; NCCL refuses two ranks on
 * one device): dlopen of libnccl.so.2 and its symbols, ncclGetUniqueId,
 * ncclCommInitRank, the three collectives the library issues (in place, on
 * a stream) and ncclCommDestroy; with one rank each collective is the
 * identity, which is checked.  Returns 0, LDA_ENCCL or LDA_ECUDA, with a
 * message in msg (msg_cap bytes). */
int lda_debug_nccl_selftest(int32_t device, char *msg, int32_t msg_cap);

/* Load this rank's documents [doc_begin, doc_end) of the global corpus,
 * randomly initialise every token's topic (L377-379; Philox at t = 0, X10)
 * and build n_wk, n_k and θ (allreduced across ranks when world > 1).
 *   doc_ptr : doc_end-doc_begin+1 offsets into `words`, doc_ptr[0] == 0,
 *             non-decreasing (empty documents are allowed)
 *   words   : doc-major token word ids, each in [0, V)
 *   seed    : 64-bit Philox key (X9)
 * Every rank must pass the same seed.  With world == 1 pass the whole corpus
 * (doc_begin = 0, doc_end = D).  Errors: LDA_EINVAL (bad ids/offsets/range),
 * LDA_ERANGE (a document longer than 65535 tokens, or >= 2^32 local tokens),
 * LDA_ENOMEM, LDA_ECUDA, LDA_ENCCL, LDA_ESTATE (called twice). */
int lda_load_corpus(lda_ctx *ctx, int64_t doc_begin, int64_t doc_end, const int64_t *doc_ptr,
                    const int32_t *words, uint64_t seed);

/* Run n_sweeps >= 0 sweeps (iterations, L415-421).  Synchronous: returns after
 * the last sweep's counts are rebuilt on every rank.  Collective when
 * world > 1.  Errors: LDA_EINVAL (n < 0), LDA_ESTATE, LDA_ECUDA, LDA_ENCCL. */
int lda_iterate(lda_ctx *ctx, int32_t n_sweeps);

/* Per-token log-likelihood of the current state (Fig. 8; formula
 * of reading X11, the collapsed joint log p(w, z | α, β) divided by the global
 * token count T).  Collective when world > 1. */
int lda_loglik(lda_ctx *ctx, double *ll_per_token);

/* Copy the model out (Alg. 1 lines 17-20, L829-835).  Any pointer may be NULL.
 *   n_wk       : V*K int32, row-major by word (X13) — global counts
 *   n_k        : K int32
 *   ndk_ptr    : D_g+1 int64 CSR offsets of θ for this rank's documents
 *   ndk_topic, ndk_count : ndk_capacity entries each; topics ascending per row
 *   ndk_nnz_out: receives Σ_d nnz_d (the capacity needed).  If ndk_topic or
 *                ndk_count is non-NULL and ndk_capacity < nnz the call writes
 *                *ndk_nnz_out and returns LDA_ERANGE.
 *   z          : T_g uint16 topics in input (doc-major) order */
int lda_get_counts(lda_ctx *ctx, int32_t *n_wk, int32_t *n_k, int64_t *ndk_ptr,
                   uint16_t *ndk_topic, int32_t *ndk_count, int64_t ndk_capacity,
                   int64_t *ndk_nnz_out, uint16_t *z);

/* Statistics of the last lda_iterate call. */
int lda_get_stats(lda_ctx *ctx, lda_stats *out);

/* Per-sweep log of the last lda_iterate call: up to `cap` entries of each
 * non-NULL array (device ms per sweep and per phase; Σ_t nnz_{d(t)} of the θ
 * each sweep sampled against; Σ_d nnz_d of the θ each sweep rebuilt).
 * *n_out = number of sweeps in that call. */
int lda_get_sweep_log(lda_ctx *ctx, int32_t cap, double *ms_sweep, double *ms_sample, double *ms_recount,
                      double *ms_theta, double *ms_allreduce, int64_t *sum_nnz_tok, int64_t *sum_nnz_doc,
                      int32_t *n_out);

/* LL/token log of the last lda_iterate call (option "loglik_every"): up to
 * `cap` entries of each non-NULL array -- the sweep counter t after which
 * it was taken and the LL/token (lda_loglik's definition).  *n_out = number
 * of entries in that call. */
int lda_get_loglik_log(lda_ctx *ctx, int32_t cap, int64_t *sweep, double *ll_per_token, int32_t *n_out);

/* The CUDA stream (cudaStream_t) the sweep kernels run on; valid after
 * lda_load_corpus until lda_destroy. */
int lda_get_stream(lda_ctx *ctx, void **stream);

/* Test hook (teacher forcing): replace every local token's topic with z
 * (T_g uint16, input order, each < K) and rebuild all counts (collective when
 * world > 1).  Does not advance the sweep counter. */
int lda_set_z(lda_ctx *ctx, const uint16_t *z);

/* Free everything (NULL is a no-op). */
void lda_destroy(lda_ctx *ctx);

/* Detail of the last failure on ctx ("" if none; a static string for NULL). */
const char *lda_last_error(const lda_ctx *ctx);

/* Library version string. */
const char *lda_version(void);

#ifdef __cplusplus
}
#endif
#endif /* LDA_H */
