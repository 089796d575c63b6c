// Internal declarations shared by the host runtime (api.cpp, host_prep.cpp)
// and the kernels (kernels.cu).  Not part of the ABI.
#pragma once

#include <cstdint>
#include <string>
#include <vector>

namespace lda {

// One sampling work item: a run of tokens of one word inside one doc tile
// (word-first order, L1189-1191; heavy words split over several items,
// L1203-1221).  c_base = canonical index (X18) of the item's first token.
struct SampleChunk {
    uint32_t begin;   // first word-major position
    uint32_t count;   // tokens
    uint32_t word;
    uint32_t pad;
    uint64_t c_base;
};

// One n_wk-recount work item: tokens [vbegin, vbegin+vcount) of word `word`
// counted across its per-tile segments.  split != 0 when the word has more
// than one item (its row is zeroed first and accumulated atomically).
struct RecountChunk {
    uint32_t word;
    uint32_t vbegin;
    uint32_t vcount;
    uint32_t split;
};

// Host-side layout of one rank's shard (built by build_layout).
struct HostLayout {
    int64_t D = 0, T = 0;
    int32_t V = 0, K = 0;
    int32_t ntiles = 1;
    std::vector<uint32_t> doc_ptr32;   // D+1 doc-major token offsets
    std::vector<uint32_t> row_off16;   // D   θ row start, in 16-byte units
    uint64_t rows16 = 0;               // θ row buffer size in 16-byte units (incl. tail pad)
    std::vector<uint32_t> tok_row;     // T   word-major: θ row (16 B units) of the token's doc
    std::vector<uint32_t> doc_map;     // T   doc-major token i -> word-major position (S7, L1297-1303)
    std::vector<uint32_t> tseg;        // ntiles*V+1 segment starts, key = tile*V + word
    std::vector<SampleChunk> chunks;   // heavy-first
    std::vector<RecountChunk> rchunks; // heavy-first
    std::vector<int32_t> split_words;  // words whose row is accumulated atomically
    std::vector<int64_t> word_count;   // V local tokens per word
};

// cbase[w] = canonical index of this rank's first token of word w.
// Returns "" on success, else an error message.
std::string build_layout(const int64_t *doc_ptr, const int32_t *words, int64_t D, int32_t V,
                         int32_t K, const int64_t *cbase, int64_t tile_tokens,
                         int64_t chunk_tokens, int64_t recount_tokens, int nthreads,
                         HostLayout &out);

// Host-side validation of a local corpus; "" if valid.  *too_long set when a
// doc exceeds 65535 tokens.
std::string validate_corpus(const int64_t *doc_ptr, const int32_t *words, int64_t D, int32_t V,
                            bool *range_error);

int host_threads(int requested);

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
    uint32_t *doc_ptr32 = nullptr;  // D+1
    uint32_t *row_off16 = nullptr;  // D
    uint32_t *tseg = nullptr;       // ntiles*V+1
    SampleChunk *chunks = nullptr;
    int64_t n_chunks = 0;
    RecountChunk *rchunks = nullptr;
    int64_t n_rchunks = 0;
    int32_t *split_words = nullptr;
    int64_t n_split = 0;
    // model
    uint32_t *rows = nullptr;       // θ rows, rows16*4 words
    int32_t *nwk = nullptr;         // V*K + K (n_k at offset V*K)
    double *invk = nullptr;         // K
    // scratch
    uint32_t *counter = nullptr;    // work counters [4]
    unsigned long long *stat = nullptr;  // [4]: Σ L_d nnz_d, Σ nnz_d
    double *ll_part = nullptr;      // partial sums
    double *ll_out = nullptr;       // [2]
    double *sweep_scratch = nullptr;  // sweep_grid*2*K when K does not fit in smem
    int num_sms = 148;
    int sweep_grid = 0;
    int theta_grid = 0, theta_block = 0;
    size_t sweep_smem = 0, theta_smem = 0;
    int ll_blocks = 0;
};

int configure_kernels(DevState &s);
int launch_init(const DevState &s, void *stream);
int launch_recount(const DevState &s, void *stream, int *launches);
int launch_theta(const DevState &s, unsigned long long *stat_out, void *stream, int *launches);
int launch_sweep(const DevState &s, uint32_t t, void *stream, int *launches);
int launch_loglik(const DevState &s, bool word_part, void *stream, int *launches);

}  // namespace lda
