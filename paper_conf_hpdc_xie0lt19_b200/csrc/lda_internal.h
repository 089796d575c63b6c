// Internal declarations shared by the host runtime (api.cpp, host_prep.cpp)
// and the kernels (kernels.cu).  Not part of the ABI.
#pragma once

#include <condition_variable>
#include <cstdint>
#include <functional>
#include <memory>
#include <mutex>
#include <string>
#include <vector>

namespace lda {

// Owning host array for the large per-token tables: uninitialised, 2 MB
// aligned with transparent huge pages requested (the layout's random
// scatters would otherwise miss the TLB on every write), first touched in
// parallel by the threads that fill it.
template <class T>
class HostBuf {
  public:
    HostBuf() = default;
    HostBuf(const HostBuf &) = delete;
    HostBuf &operator=(const HostBuf &) = delete;
    ~HostBuf() { release(); }
    bool allocate(size_t n);   // defined in host_prep.cpp (explicit instantiations)
    void release();
    T *data() { return p_; }
    const T *data() const { return p_; }
    size_t size() const { return n_; }
    T &operator[](size_t i) { return p_[i]; }
    const T &operator[](size_t i) const { return p_[i]; }

  private:
    T *p_ = nullptr;
    size_t n_ = 0;
};

// A run of word w's tokens inside one document tile.  Word w's local tokens
// have "virtual" indices 0..n_w-1 in (doc, position) order, i.e. canonical
// order (X18) restricted to this rank; the run stores virtual indices
// [vstart, next.vstart) at word-major positions pos, pos+1, ...  Each word's
// runs are followed by a sentinel {0, n_w}.
struct Seg {
    uint32_t pos;
    uint32_t vstart;
};

// One sampling work item: tokens [vbegin, vbegin+count) of one word (the
// word-first order of L1189-1191; heavy words split over several items,
// L1203-1221).  Runs [seg0, segN) hold the item (segN = the word's
// sentinel); c_base = canonical index of the rank's first token of the word
// (a token's index is c_base + tok_crank[p]).
struct SampleChunk {
    uint32_t word;
    uint32_t vbegin;
    uint32_t count;
    uint32_t seg0;
    uint32_t segN;
    uint32_t pad;
    uint64_t c_base;
};

// One n_wk-recount work item: virtual indices [vbegin, vbegin+vcount) of word
// (word & 0x7fffffff); bit 31 set when the word has more than one item (its
// row is then zeroed first and accumulated atomically).
struct RecountChunk {
    uint32_t word;
    uint32_t vbegin;
    uint32_t vcount;
    uint32_t seg0;
    uint32_t segN;
    uint32_t pad[3];
};

// Tile sampler (sweep_tile_kernel) work item: the tokens of one word inside
// one document tile -- contiguous word-major positions [pos, pos + n) --
// or a piece of them (at most chunk_tokens).  Items are queued tile by tile.
struct TileItem {
    uint32_t word;
    uint32_t pos;
    uint32_t n;
    uint32_t crank0;  // canonical rank (within the word, this rank) of the item's first token;
                      // the run holds the word's tokens in canonical order: token pos + j has crank0 + j
};

// Host-side layout of one rank's shard (built by build_layout).
struct HostLayout {
    int64_t D = 0, T = 0;
    int32_t V = 0, K = 0;
    int32_t ntiles = 1;
    std::vector<uint32_t> doc_ptr32;   // D+1 doc-major token offsets
    std::vector<uint32_t> row_off32;   // D   θ row start, in 32-byte units
    uint64_t rows32 = 0;               // θ row buffer size in 32-byte units (incl. tail pad)
    HostBuf<uint32_t> tok_row;         // T   word-major: θ row (32 B units) of the token's doc
    HostBuf<uint32_t> doc_map;         // T   doc-major token i -> word-major position (S7, L1297-1303)
    HostBuf<uint32_t> tok_crank;       // T   word-major: canonical rank of the token within its word
    std::vector<Seg> segs;             // per word: its runs, then a sentinel
    std::vector<SampleChunk> chunks;   // heavy-first
    std::vector<RecountChunk> rchunks; // heavy-first
    std::vector<int32_t> split_words;  // words whose row is accumulated atomically (recount)
    std::vector<int32_t> zero_words;   // words split over sampler chunks or without tokens
    std::vector<int64_t> word_count;   // V local tokens per word
    std::vector<TileItem> titems;      // tile sampler items: tile-major, heavy-first inside a tile
    // device_scatter only: the document tiles and the tail words (the sort key of layout_gpu.cu)
    std::vector<uint32_t> tile_doc;    // ndt+1 document boundaries of the document tiles
    std::vector<uint8_t> tail;         // V: 1 = the word's tokens form one run in the tail tile
};

// cbase[w] = canonical index of this rank's first token of word w.
// on_final(pos_begin, pos_end, tok_begin, tok_end), if set, is called as soon
// as tok_row / tok_crank over word-major positions [pos_begin, pos_end) and
// doc_map over document-major tokens [tok_begin, tok_end) are final (after
// each document tile, and for the tail region at the end) -- the caller can
// start their host->device copies while the next tile is prepared.
// Returns "" on success, else an error message ("invalid: ..." for an invalid
// corpus: a word id outside [0, V) when word_counts is null and the layout
// validated the ids itself; anything else is a range error).
std::string build_layout(const int64_t *doc_ptr, const int32_t *words, int64_t D, int32_t V,
                         int32_t K, const int64_t *cbase, int64_t tile_tokens,
                         int64_t chunk_tokens, int64_t recount_tokens, int nthreads,
                         int sampler, int64_t tail_per_tile, HostLayout &out,
                         const std::function<void(uint64_t, uint64_t, uint64_t, uint64_t)> &on_final = {},
                         const int64_t *word_counts = nullptr,  // V local tokens per word, if known
                         bool host_tok_row = true,   // tile layout: false = tok_row left to the device (launch_tok_row)
                         bool device_scatter = false,   // tile layout: doc_map left to the device (layout_gpu.cu)
                         // device_scatter: called once L.doc_ptr32, L.tile_doc and L.tail are final
                         // (the device sort of the tokens can start while the host builds the rest)
                         const std::function<void()> &on_keys = {});

// Host-side validation of a local corpus; "" if valid.  *too_long set when a
// doc exceeds 65535 tokens.
std::string validate_corpus(const int64_t *doc_ptr, const int32_t *words, int64_t D, int32_t V,
                            bool *range_error, int64_t *word_counts = nullptr,  // V counts, if wanted
                            int nthreads = 0,                                     // 0: all host threads
                            bool check_words = true);  // false: offsets and sizes only (the layout checks the ids)

int host_threads(int requested);

// out[w] = number of tokens of word w (parallel over host threads).
void word_histogram(const int32_t *words, int64_t T, int32_t V, int nthreads, int64_t *out);

// Phase timer for corpus loading: prints "[lda] <what> <ms>" to stderr when
// the environment variable LDA_TIMING is set (diagnostics only).
void tmark(const char *what);

// ---------------------------------------------------------------------------
// Kernel launchers (kernels.cu).  All return cudaError_t as int.
// ---------------------------------------------------------------------------
struct DevState {
    int32_t V = 0, K = 0;
    int64_t D = 0, T = 0;
    int32_t ntiles = 1;
    double alpha = 0, beta = 0;
    uint64_t seed = 0;
    int exclude_self = 0;
    // corpus
    uint32_t *tok_row = nullptr;    // T
    uint16_t *tok_z = nullptr;      // T (word-major)
    uint32_t *doc_map = nullptr;    // T
    uint32_t *tok_crank = nullptr;  // T (word-major); null for the tile samplers (ranks from the items)
    uint16_t *z_doc = nullptr;      // T, z in document order (θ rebuild, phase A)
    uint32_t *doc_ptr32 = nullptr;  // D+1
    uint32_t *row_off32 = nullptr;  // D
    Seg *segs = nullptr;
    SampleChunk *chunks = nullptr;
    int64_t n_chunks = 0;
    RecountChunk *rchunks = nullptr;
    int64_t n_rchunks = 0;
    int32_t *split_words = nullptr;
    int64_t n_split = 0;
    TileItem *titems = nullptr;     // tile sampler items
    int64_t n_titems = 0;
    uint64_t *cbase = nullptr;      // V: canonical index of the rank's first token of each word
    // model
    uint32_t *rows = nullptr;       // θ rows, rows32*8 words
    uint64_t rows32 = 0;            // θ row storage in 32-byte units; the last 4 (one 128-byte line) stay zero
    int32_t *nwk = nullptr;         // V*K + K (n_k at offset V*K), the current counts
    int32_t *nwk_alt = nullptr;     // the other buffer: the sampler's fused recount writes here
    int32_t *zero_words = nullptr;  // words whose next-n_wk row is zeroed before the sweep
    int64_t n_zero_words = 0;
    bool sweep_fused = false;
    int sampler = -1;               // option: -1 auto, 2 = tile sampler, 3 = its CTA form, 0 = lane-per-token
    bool sweep_tile = false;        // the tile sampler is used (sampler 2, fits in smem, no exclude_self)
    bool sweep_tile_cta = false;    // its large-K form with CTA-shared tables (sampler 3)
    bool tile_cta_gnk = false;      // ... with n_k by global reductions and compact tables (K > kTileMaxK)
    int tile_nbuf = 2;              // ... its table buffers per CTA
    bool tile_fused = true;         // option fused_recount: the tile samplers update n_wk / n_k themselves
    size_t tile_smem = 0;
    int tile_grid = 0, tile_block = 0, tile_lmax = 160;
    char *wtab = nullptr;           // tile sampler: per-word tables (p32, dense prefix), rebuilt every sweep
    size_t wt_bytes = 0;
    // f2, sampler 3 with compact tables: sparse word rows (kernels.cu SparseRows)
    uint32_t *sp_off = nullptr;     // V+1: word w's entries [sp_off[w], sp_off[w+1]) (empty: a dense table)
    uint32_t *sp_nnz = nullptr;     // V: its nonzero topics this sweep
    uint32_t *sp_ent = nullptr;     // 2 words per entry (topic, fp32 p* bits)
    float *s32 = nullptr;           // K4: the smoothing row fl32(β / (n_k + Vβ))
    int64_t sp_words = 0;           // words with sparse rows
    int64_t sp_cap = 0;             // entries allocated
    double certify_slack = 1.0;     // test option: scales the tile sampler's certification bounds
    double *denom = nullptr;        // K: n_k + Vβ of the frozen counts
    // scratch
    uint32_t *counter = nullptr;    // work counters [4]
    unsigned long long *stat = nullptr;  // [4]: Σ L_d nnz_d, Σ nnz_d
    double *ll_part = nullptr;      // partial sums
    double *ll_out = nullptr;       // [2]
    double *sweep_scratch = nullptr;  // sweep_grid*2*K when K does not fit in smem
    int num_sms = 148;
    int sweep_grid = 0, sweep_block = 0;
    int theta_grid = 0, theta_block = 0;
    bool recount_gmem = false, theta_gmem = false;  // K > 16384: K-length histograms in global scratch
    int recount_bps = 8;                            // recount CTAs per SM (8: 2.06 -> 1.11 ms at PubMed shape vs 4)
    int *recount_scratch = nullptr;                 // recount_gmem: num_sms*recount_bps CTAs x 2K
    uint32_t *theta_scratch = nullptr;              // theta_gmem: theta_grid*8 warps x (K + K/32)
    size_t sweep_smem = 0, theta_smem = 0;
    int ll_blocks = 0;
};

int configure_kernels(DevState &s);
int launch_init(const DevState &s, void *stream);
// tok_row[doc_map[i]] = row_off32[d(i)] on the device (the tile layout's host pass leaves it out)
int launch_tok_row(const DevState &s, void *stream);
int launch_recount(const DevState &s, void *stream, int *launches, int64_t rc0 = 0, int64_t rc1 = -1,
                   bool first = true);
int launch_theta(const DevState &s, unsigned long long *stat_out, void *stream, int *launches);
// z in document order <-> word-major, through doc_map (device buffers of T entries; zd 16-byte aligned)
int launch_gather_z(const DevState &s, uint16_t *zd, void *stream);
int launch_scatter_z(const DevState &s, const uint16_t *zd, void *stream);
// parts: bit 0 = prologue + per-word tables (once per sweep), bit 1 = the
// sampling kernel (tile samplers; sampler 0 always runs both)
int launch_sweep(const DevState &s, uint32_t t, void *stream, int *launches, void *table_done_event,
                 int parts = 3);
int launch_loglik(const DevState &s, bool word_part, void *stream, int *launches);

// layout_gpu.cu: the doc-word map of the tile layout built on the device.
// keys[i] = (tail[w] ? ndt : tile(d(i)))·V + w, vals[i] = i for every token i
// (keys may alias words)
int launch_layout_keys(const uint32_t *doc_ptr32, const int32_t *words, const uint8_t *tail, const uint32_t *tile_doc,
                       int ndt, int32_t V, int64_t D, uint32_t *keys, uint32_t *vals, int num_sms, void *stream);
// stable LSD radix sort of (keys, vals) by the low `bits` key bits (8 per
// pass); the result is in (keys_tmp, vals_tmp) when *result_in_tmp, else in
// (keys, vals); temp: radix_sort_temp_words(n) words
size_t radix_sort_temp_words(uint64_t n);
int radix_sort_pairs(uint32_t *keys, uint32_t *vals, uint32_t *keys_tmp, uint32_t *vals_tmp, uint64_t n, int bits,
                     uint32_t *temp, void *stream, bool *result_in_tmp);
// doc_map[vals[p]] = p
int launch_invert(const uint32_t *vals, uint32_t *doc_map, uint64_t n, void *stream);

// ---------------------------------------------------------------------------
// The exchange of Eq. 4 (L935-937), comm.cpp.  All calls return an lda_status
// and fill `err` on failure.  Buffers are device pointers on the rank's GPU;
// `stream` is the stream after which the buffer is final (NCCL enqueues on
// it; the peer backend synchronises it and returns with the result written).
// ---------------------------------------------------------------------------
constexpr int kMaxPeers = 16;

class Comm {
  public:
    virtual ~Comm() = default;
    virtual const char *name() const = 0;
    virtual int allreduce_i32(int32_t *buf, size_t n, void *stream, std::string &err) = 0;  // in place, sum
    virtual int allreduce_f64(double *buf, size_t n, void *stream, std::string &err) = 0;   // in place, sum
    // recv[q*n .. (q+1)*n) = rank q's send[0 .. n)
    virtual int allgather_i64(const int64_t *send, int64_t *recv, size_t n, void *stream, std::string &err) = 0;
    int rank() const { return rank_; }
    int world() const { return world_; }

  protected:
    int rank_ = 0, world_ = 1;
};

// In-process group of `world` ranks, each driven by its own host thread.
class PeerGroup {
  public:
    explicit PeerGroup(int world);
    int world() const { return world_; }
    int join(int rank, int device, std::string &err);
    int barrier(std::string &err);
    void set_ptr(int rank, void *p);
    void ptrs(void **out);
    int device(int rank);
    void mark_broken();

  private:
    int world_;
    std::mutex mu_;
    std::condition_variable cv_;
    int arrived_ = 0;
    uint64_t gen_ = 0;
    bool broken_ = false;
    int timeout_s_ = 600;
    std::vector<void *> ptr_;
    std::vector<int> dev_;
    std::vector<int> joined_;
};

int nccl_unique_id(void *out128, std::string &err);
int make_nccl_comm(int rank, int world, const void *uid, int device, std::unique_ptr<Comm> &out, std::string &err);
int make_peer_comm(const std::shared_ptr<PeerGroup> &g, int rank, int device, std::unique_ptr<Comm> &out,
                   std::string &err);

// Peer-memory collective kernels (kernels.cu).  ptrs[q] = rank q's buffer of
// n elements of esz bytes (4: int32, 8: fp64 when is_f64).  Slice q is
// [lo(q), lo(q+1)) with lo(q) = 16-byte-aligned q·n/world.
// reduce-scatter: own[slice rank] = Σ_q ptrs[q][slice rank] (rank order);
// all-gather: own[slice q] = ptrs[q][slice q] for every q != rank.
int launch_peer_reduce_scatter(void *const *ptrs, int world, int rank, void *own, size_t n, size_t esz, int is_f64,
                               void *stream);
int launch_peer_all_gather(void *const *ptrs, int world, int rank, void *own, size_t n, size_t esz, void *stream);

}  // namespace lda
