// Host-side corpus preparation (the paper's CPU preprocessing, L593-597):
// validation, the word-first token order (L1189-1191), the document-word map
// (L1297-1303), fixed-capacity θ rows (CSR with short column index,
// L1235-1243) and the heavy-first work-item tables (L1203-1221).
#include <atomic>
#include <sys/mman.h>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <thread>

#include "lda_internal.h"

namespace lda {

template <class T>
bool HostBuf<T>::allocate(size_t n) {
    release();
    const size_t align = size_t(2) << 20;
    const size_t bytes = (std::max<size_t>(n, 1) * sizeof(T) + align - 1) / align * align;
    void *q = std::aligned_alloc(align, bytes);
    if (!q) return false;
#ifdef MADV_HUGEPAGE
    madvise(q, bytes, MADV_HUGEPAGE);
#endif
    p_ = static_cast<T *>(q);
    n_ = n;
    return true;
}
template <class T>
void HostBuf<T>::release() {
    std::free(p_);
    p_ = nullptr;
    n_ = 0;
}
template class HostBuf<uint32_t>;

void tmark(const char *what) {
    static const bool on = std::getenv("LDA_TIMING") != nullptr;
    static auto last = std::chrono::steady_clock::now();
    const auto now = std::chrono::steady_clock::now();
    if (on && what)
        std::fprintf(stderr, "[lda] %-28s %9.1f ms\n", what,
                     std::chrono::duration<double, std::milli>(now - last).count());
    last = now;
}

int host_threads(int requested) {
    unsigned hw = std::thread::hardware_concurrency();
    if (hw == 0) hw = 1;
    int n = requested > 0 ? requested : static_cast<int>(hw);
    return std::max(1, std::min(n, 64));
}

// f(thread_id, begin, end) over [0, n) split into nthreads contiguous parts.
template <class F>
static void parallel_for(int nthreads, int64_t n, F f) {
    if (nthreads <= 1 || n < (1 << 16)) {
        f(0, int64_t(0), n);
        return;
    }
    std::vector<std::thread> th;
    th.reserve(nthreads);
    for (int t = 0; t < nthreads; ++t) {
        int64_t b = n * t / nthreads, e = n * (t + 1) / nthreads;
        th.emplace_back([=, &f] { f(t, b, e); });
    }
    for (auto &x : th) x.join();
}

void word_histogram(const int32_t *words, int64_t T, int32_t V, int nthreads, int64_t *out) {
    nthreads = host_threads(nthreads);
    const int nth = T < (1 << 16) ? 1 : nthreads;
    std::vector<std::vector<uint32_t>> h(nth, std::vector<uint32_t>(V, 0u));
    std::vector<std::thread> th;
    auto part = [&](int t) {
        auto &hh = h[t];
        const int64_t b = T * t / nth, e = T * (t + 1) / nth;
        for (int64_t i = b; i < e; ++i) hh[words[i]]++;
    };
    for (int t = 1; t < nth; ++t) th.emplace_back(part, t);
    part(0);
    for (auto &x : th) x.join();
    for (int32_t w = 0; w < V; ++w) {
        int64_t s = 0;
        for (int t = 0; t < nth; ++t) s += h[t][w];
        out[w] = s;
    }
}

std::string validate_corpus(const int64_t *doc_ptr, const int32_t *words, int64_t D, int32_t V,
                            bool *range_error, int64_t *word_counts, int nthreads, bool check_words) {
    *range_error = false;
    if (D < 0) return "negative document count";
    if (!doc_ptr) return "doc_ptr is NULL";
    if (doc_ptr[0] != 0) return "doc_ptr[0] must be 0";
    for (int64_t d = 0; d < D; ++d) {
        int64_t len = doc_ptr[d + 1] - doc_ptr[d];
        if (len < 0) return "doc_ptr must be non-decreasing";
        if (len > 65535) {
            *range_error = true;
            return "document " + std::to_string(d) + " has " + std::to_string(len) +
                   " tokens (> 65535, the uint16 θ count limit)";
        }
    }
    int64_t T = doc_ptr[D];
    if (T >= (int64_t(1) << 32)) {
        *range_error = true;
        return "more than 2^32-1 tokens on one rank";
    }
    if (T > 0 && !words) return "words is NULL";
    if (!check_words) return "";
    int nth = host_threads(nthreads);
    std::vector<int64_t> bad(nth, -1);
    // with word_counts: the same pass counts the tokens of every word
    const int nparts = T < (1 << 16) ? 1 : nth;
    std::vector<std::vector<uint32_t>> h(word_counts ? nparts : 0, std::vector<uint32_t>(V, 0u));
    parallel_for(nth, T, [&](int t, int64_t b, int64_t e) {
        uint32_t *hh = word_counts ? h[t].data() : nullptr;
        for (int64_t i = b; i < e; ++i) {
            const int32_t w = words[i];
            if (w < 0 || w >= V) {
                bad[t] = i;
                return;
            }
            if (hh) hh[w]++;
        }
    });
    for (int64_t i : bad)
        if (i >= 0)
            return "word id " + std::to_string(words[i]) + " at token " + std::to_string(i) +
                   " outside [0, V)";
    if (word_counts)
        for (int32_t w = 0; w < V; ++w) {
            int64_t c = 0;
            for (const auto &hh : h) c += hh[w];
            word_counts[w] = c;
        }
    return "";
}

std::string build_layout(const int64_t *doc_ptr, const int32_t *words, int64_t D, int32_t V,
                         int32_t K, const int64_t *cbase, int64_t tile_tokens,
                         int64_t chunk_tokens, int64_t recount_tokens, int nthreads,
                         int sampler, int64_t tail_per_tile, HostLayout &L,
                         const std::function<void(uint64_t, uint64_t, uint64_t, uint64_t)> &on_final,
                         const int64_t *word_counts, bool host_tok_row, bool device_scatter,
                         const std::function<void()> &on_keys) {
    const int64_t T = doc_ptr[D];
    L.D = D;
    L.T = T;
    L.V = V;
    L.K = K;
    nthreads = host_threads(nthreads);

    // θ rows: 1 header word (nnz) + capacity min(L_d, K) entries, rounded up
    // to whole 128-byte lines (the tile samplers read a row line by line);
    // words past nnz are kept zero (zero-mass padding the sampler reads
    // without a bounds check).  Offsets are in 32-byte units.
    L.doc_ptr32.resize(D + 1);
    L.row_off32.resize(D);
    uint64_t off32 = 0;
    for (int64_t d = 0; d < D; ++d) {
        int64_t len = doc_ptr[d + 1] - doc_ptr[d];
        int64_t cap = std::min<int64_t>(len, K);
        L.doc_ptr32[d] = static_cast<uint32_t>(doc_ptr[d]);
        L.row_off32[d] = static_cast<uint32_t>(off32);
        off32 += 4 * static_cast<uint64_t>((cap + 1 + 31) / 32);
        if (off32 >= (uint64_t(1) << 32) - 64) return "θ row storage exceeds 2^32 x 32 bytes";
        // the tile samplers' line tables flag a row's first line in bit 31
        if (sampler == 2 && off32 >= (uint64_t(1) << 31) - 64)
            return "θ row storage exceeds 2^31 x 32 bytes (64 GB) on one rank: use more ranks or sampler 0";
    }
    L.doc_ptr32[D] = static_cast<uint32_t>(T);
    L.rows32 = off32 + 4;  // tail pad

    // Doc tiles: contiguous document ranges of about tile_tokens tokens.
    std::vector<int64_t> tile_doc{0};
    if (tile_tokens > 0) {
        int64_t acc = 0;
        for (int64_t d = 0; d < D; ++d) {
            int64_t len = doc_ptr[d + 1] - doc_ptr[d];
            if (acc > 0 && acc + len > tile_tokens) {
                tile_doc.push_back(d);
                acc = 0;
            }
            acc += len;
        }
    }
    tile_doc.push_back(D);
    const int ndt = static_cast<int>(tile_doc.size()) - 1;  // document tiles

    // Word counts of the shard.  Without word_counts the word ids are also
    // validated here (the caller skipped its own pass over the words): by
    // the per-tile counts of the thread-per-tile pass below, or one parallel
    // histogram.
    const bool tile_fast = sampler == 2 && ndt >= 2 * nthreads;  // one host thread per tile (see below)
    std::vector<int64_t> wc(V, 0);
    std::vector<std::vector<uint32_t>> pre_cnt;  // tile_fast: the doc tiles' word counts
    if (word_counts) {
        std::copy(word_counts, word_counts + V, wc.begin());
    } else if (tile_fast) {
        pre_cnt.resize(ndt);
        std::atomic<int> next_tile{0};
        std::atomic<int64_t> bad{-1};
        std::vector<std::thread> th;
        auto count = [&] {
            for (int b; (b = next_tile.fetch_add(1)) < ndt;) {
                auto &tc = pre_cnt[b];
                tc.assign(V, 0);
                const int64_t i1 = doc_ptr[tile_doc[b + 1]];
                for (int64_t i = doc_ptr[tile_doc[b]]; i < i1; ++i) {
                    const uint32_t w = static_cast<uint32_t>(words[i]);
                    if (w >= static_cast<uint32_t>(V)) {
                        bad = i;
                        break;
                    }
                    tc[w]++;
                }
            }
        };
        for (int t = 1; t < nthreads; ++t) th.emplace_back(count);
        count();
        for (auto &x : th) x.join();
        if (bad >= 0)
            return "invalid: word id " + std::to_string(words[bad.load()]) + " at token " +
                   std::to_string(bad.load()) + " outside [0, V)";
        parallel_for(nthreads, V, [&](int, int64_t w0, int64_t w1) {
            for (int64_t w = w0; w < w1; ++w) {
                int64_t c = 0;
                for (int b = 0; b < ndt; ++b) c += pre_cnt[b][w];
                wc[w] = c;
            }
        });
    } else {
        bool range_err = false;
        std::string v = validate_corpus(doc_ptr, words, D, V, &range_err, wc.data(), nthreads);
        if (!v.empty()) return "invalid: " + v;
    }
    L.word_count = wc;

    // Tail words (tile sampler only): words with too few tokens per document
    // tile to amortise a per-(word, tile) work item get one corpus-wide run
    // in an extra "tail tile" after the document tiles.
    std::vector<uint8_t> tail(V, 0);
    bool any_tail = false;
    if (sampler == 2 && ndt > 1 && tail_per_tile > 0)
        for (int32_t w = 0; w < V; ++w)
            if (wc[w] > 0 && wc[w] < tail_per_tile * ndt) {
                tail[w] = 1;
                any_tail = true;
            }
    const int nt = ndt + (any_tail ? 1 : 0);
    L.ntiles = nt;

    // Tile samplers: documents keep their order inside each tile part, so a
    // word's run holds its tokens in canonical order and a token's rank is
    // its item's base + offset (no per-token rank table).  Sampler 0:
    // documents by decreasing length inside a part (similar θ row lengths in
    // a warp), ranks stored per token.
    const bool tile_layout = sampler == 2;
    // tile layout: the rows of the tokens (a random 4-byte scatter over the
    // word-major stream, the costliest part of the host pass) are left to
    // the device unless asked for (launch_tok_row from doc_map)
    const bool want_row = !tile_layout || host_tok_row;
    // device_scatter (tile layout): the per-token scatter -- doc_map -- is left
    // to the device (layout_gpu.cu), which sorts the tokens by the key
    // tile·V + word (tail words: ndt·V + word); the host keeps the counts
    const bool dev_scatter = device_scatter && tile_layout && !want_row;
    if ((want_row && !L.tok_row.allocate(T)) || (!dev_scatter && !L.doc_map.allocate(T)) ||
        (!tile_layout && !L.tok_crank.allocate(T)))
        return "host allocation of the token tables failed";
    if (dev_scatter) {
        L.tile_doc.assign(tile_doc.begin(), tile_doc.end());
        L.tail.assign(tail.begin(), tail.end());
        // the device sort can start now (doc_ptr32, tile_doc and tail are final)
        if (on_keys) on_keys();
    }
    HostBuf<uint32_t> ctmp;  // canonical rank of token i (document order)
    if (!tile_layout && !ctmp.allocate(T)) return "host allocation of the token tables failed";
    // first touch in parallel, one store per 4 KB page (the kernel zeroes
    // the pages; every entry is written below).  Not needed when only
    // doc_map is built: the tile pass writes it in order, part by part, in
    // parallel.
    if (want_row || !tile_layout) parallel_for(nthreads, T, [&](int, int64_t b, int64_t e) {
        for (int64_t i = b; i < e; i += 1024) {
            if (want_row) L.tok_row[i] = 0u;
            L.doc_map[i] = 0u;
            if (!tile_layout) {
                L.tok_crank[i] = 0u;
                ctmp[i] = 0u;
            }
        }
    });
    tmark("layout: host tables");
    std::vector<uint32_t> tseg(static_cast<size_t>(nt) * V, 0);  // run start of (tile, word)
    std::vector<std::vector<uint32_t>> tile_cnt(nt);
    // tail region: after every document tile's segment, word by word
    int64_t tail_tokens = 0;
    for (int32_t w = 0; w < V; ++w)
        if (tail[w]) tail_tokens += wc[w];
    std::vector<uint32_t> tail_next(V, 0);  // next free position of each tail word
    {
        uint64_t tp = static_cast<uint64_t>(T - tail_tokens);
        if (any_tail) tile_cnt[ndt].assign(V, 0);
        for (int32_t w = 0; w < V; ++w)
            if (tail[w]) {
                tail_next[w] = static_cast<uint32_t>(tp);
                tseg[static_cast<size_t>(ndt) * V + w] = static_cast<uint32_t>(tp);
                tile_cnt[ndt][w] = static_cast<uint32_t>(wc[w]);
                tp += wc[w];
            }
    }
    std::vector<uint32_t> crank_run(V, 0);   // tokens of each word in earlier tiles (canonical order)
    std::vector<uint32_t> tcrank(static_cast<size_t>(nt) * V, 0);  // rank of a (tile, word) run's first token
    std::vector<std::vector<uint32_t>> cnt(nthreads, std::vector<uint32_t>(V));
    std::vector<std::vector<uint32_t>> pnext(nthreads, std::vector<uint32_t>(V));
    std::vector<std::vector<uint32_t>> cnext(nthreads, std::vector<uint32_t>(V));

    uint64_t pos = 0;  // start of the current tile's segment
    if (tile_fast) {
        // Many tiles (PubMed shape: 54 on 16 host threads): one thread per
        // tile instead of every tile split over all threads, so the per-word
        // work (V-length count arrays, their sums and prefixes) is done once
        // per tile instead of once per tile and thread.
        //   1. counts of every tile (head and tail words)
        //   2. canonical ranks of the runs (prefix over the tiles, per word),
        //      the tiles' segment starts and the head words' run starts
        //   3. the scatter, tile by tile, each tile's part announced to the
        //      copier (on_final) as soon as it is written
        std::vector<int64_t> headT(ndt, 0);
        std::atomic<int> next_tile{0};
        auto tile_threads = [&](auto &&f) {
            std::vector<std::thread> th;
            for (int t = 1; t < nthreads; ++t) th.emplace_back(f);
            f();
            for (auto &x : th) x.join();
        };
        tile_threads([&] {
            for (int b; (b = next_tile.fetch_add(1)) < ndt;) {
                auto &tc = tile_cnt[b];
                const int64_t i0 = doc_ptr[tile_doc[b]], i1 = doc_ptr[tile_doc[b + 1]];
                if (!pre_cnt.empty()) {
                    tc.swap(pre_cnt[b]);  // counted (and validated) above
                } else {
                    tc.assign(V, 0);
                    for (int64_t i = i0; i < i1; ++i) tc[words[i]]++;
                }
                int64_t tt = 0;
                for (int32_t w = 0; w < V; ++w)
                    if (tail[w]) tt += tc[w];
                headT[b] = (i1 - i0) - tt;
            }
        });
        std::vector<uint64_t> pos_tile(ndt + 1, 0);
        for (int b = 0; b < ndt; ++b) pos_tile[b + 1] = pos_tile[b] + static_cast<uint64_t>(headT[b]);
        // per word: the run's canonical rank in each tile = tokens of the word in earlier tiles
        parallel_for(nthreads, V, [&](int, int64_t w0, int64_t w1) {
            for (int64_t w = w0; w < w1; ++w) {
                uint32_t run_c = 0;
                for (int b = 0; b < ndt; ++b) {
                    tcrank[static_cast<size_t>(b) * V + w] = run_c;
                    run_c += tile_cnt[b][w];
                }
            }
        });
        next_tile = 0;
        tile_threads([&] {
            std::vector<uint32_t> next(V);
            for (int b; (b = next_tile.fetch_add(1)) < ndt;) {
                auto &tc = tile_cnt[b];
                uint32_t *tseg_b = tseg.data() + static_cast<size_t>(b) * V;
                const uint32_t *tcr_b = tcrank.data() + static_cast<size_t>(b) * V;
                uint64_t p = pos_tile[b];
                for (int32_t w = 0; w < V; ++w) {
                    if (tail[w]) {
                        // the tail word's tokens of this tile continue its tail run
                        next[w] = tail_next[w] + tcr_b[w];
                        tc[w] = 0;  // counted in the tail tile only
                    } else {
                        tseg_b[w] = static_cast<uint32_t>(p);
                        next[w] = static_cast<uint32_t>(p);
                        p += tc[w];
                    }
                }
                const int64_t d0 = tile_doc[b], d1 = tile_doc[b + 1];
                if (dev_scatter) continue;
                if (want_row) {
                    for (int64_t d = d0; d < d1; ++d) {
                        const uint32_t row = L.row_off32[d];
                        for (int64_t i = doc_ptr[d]; i < doc_ptr[d + 1]; ++i) {
                            const uint32_t q = next[words[i]]++;
                            L.doc_map[i] = q;
                            L.tok_row[q] = row;
                        }
                    }
                } else {
                    for (int64_t i = doc_ptr[d0]; i < doc_ptr[d1]; ++i) L.doc_map[i] = next[words[i]]++;
                }
                if (on_final)
                    on_final(pos_tile[b], pos_tile[b + 1], static_cast<uint64_t>(doc_ptr[d0]),
                             static_cast<uint64_t>(doc_ptr[d1]));
            }
        });
        pos = pos_tile[ndt];
    }
    for (int b = 0; b < ndt && !tile_fast; ++b) {
        const uint64_t pos_tile = pos;
        const int64_t d0 = tile_doc[b], d1 = tile_doc[b + 1];
        // the tile's documents in nth contiguous parts (original order), balanced by tokens
        const int nth = (doc_ptr[d1] - doc_ptr[d0]) < (1 << 16) ? 1 : nthreads;
        std::vector<int64_t> tdoc(nth + 1);
        tdoc[0] = d0;
        for (int t = 1; t < nth; ++t) {
            const int64_t target = doc_ptr[d0] + (doc_ptr[d1] - doc_ptr[d0]) * t / nth;
            tdoc[t] = std::max(tdoc[t - 1], std::lower_bound(doc_ptr + d0, doc_ptr + d1, target) - doc_ptr);
        }
        tdoc[nth] = d1;
        auto run_parts = [&](auto &&f) {
            std::vector<std::thread> th;
            for (int t = 1; t < nth; ++t) th.emplace_back(f, t);
            f(0);
            for (auto &x : th) x.join();
        };
        // count (all words)
        run_parts([&](int t) {
            auto &h = cnt[t];
            std::fill(h.begin(), h.end(), 0u);
            for (int64_t i = doc_ptr[tdoc[t]]; i < doc_ptr[tdoc[t + 1]]; ++i) h[words[i]]++;
        });
        // bases: word-major positions (head words: this tile's segment; tail
        // words: their tail run) and canonical ranks, part by part
        // (in parallel over word ranges: the tile's tokens of each word, the
        // head words' segment starts by a serial prefix over the words, then
        // every word's run start per part)
        auto &tc = tile_cnt[b];
        tc.assign(V, 0);
        auto word_parts = [&](auto &&f) {
            run_parts([&](int t) {
                f(static_cast<int32_t>(static_cast<int64_t>(V) * t / nth),
                  static_cast<int32_t>(static_cast<int64_t>(V) * (t + 1) / nth));
            });
        };
        uint32_t *tseg_b = tseg.data() + static_cast<size_t>(b) * V;
        word_parts([&](int32_t w0, int32_t w1) {
            for (int32_t w = w0; w < w1; ++w) {
                if (tail[w]) continue;
                uint32_t n = 0;
                for (int t = 0; t < nth; ++t) n += cnt[t][w];
                tc[w] = n;
            }
        });
        for (int32_t w = 0; w < V; ++w)
            if (!tail[w]) {
                tseg_b[w] = static_cast<uint32_t>(pos);
                pos += tc[w];
            }
        word_parts([&](int32_t w0, int32_t w1) {
            for (int32_t w = w0; w < w1; ++w) {
                uint32_t run_p = tail[w] ? tail_next[w] : tseg_b[w];
                uint32_t run_c = crank_run[w];
                tcrank[static_cast<size_t>(b) * V + w] = run_c;
                for (int t = 0; t < nth; ++t) {
                    const uint32_t h = cnt[t][w];
                    pnext[t][w] = run_p;
                    cnext[t][w] = run_c;
                    run_p += h;
                    run_c += h;
                }
                crank_run[w] = run_c;
                if (tail[w]) tail_next[w] = run_p;
            }
        });
        // scatter: canonical ranks in document order, then positions with the
        // part's documents by decreasing length, so that the 32 tokens a warp
        // draws together (consecutive in a word's run) come from documents of
        // similar length -> similar θ row lengths -> little SIMT divergence.
        // (The Philox counter does not depend on this order: each token
        // carries its canonical rank.)
        if (!dev_scatter) run_parts([&](int t) {
            auto &next = pnext[t];
            if (tile_layout && !want_row) {
                for (int64_t i = doc_ptr[tdoc[t]]; i < doc_ptr[tdoc[t + 1]]; ++i) L.doc_map[i] = next[words[i]]++;
                return;
            }
            if (tile_layout) {
                for (int64_t d = tdoc[t]; d < tdoc[t + 1]; ++d) {
                    const uint32_t row = L.row_off32[d];
                    for (int64_t i = doc_ptr[d]; i < doc_ptr[d + 1]; ++i) {
                        const uint32_t p = next[words[i]]++;
                        L.doc_map[i] = p;
                        L.tok_row[p] = row;
                    }
                }
                return;
            }
            auto &cn = cnext[t];
            for (int64_t i = doc_ptr[tdoc[t]]; i < doc_ptr[tdoc[t + 1]]; ++i) ctmp[i] = cn[words[i]]++;
            std::vector<int64_t> ord(tdoc[t + 1] - tdoc[t]);
            for (size_t k = 0; k < ord.size(); ++k) ord[k] = tdoc[t] + static_cast<int64_t>(k);
            std::stable_sort(ord.begin(), ord.end(), [&](int64_t x, int64_t y) {
                return doc_ptr[x + 1] - doc_ptr[x] > doc_ptr[y + 1] - doc_ptr[y];
            });
            for (const int64_t d : ord) {
                const uint32_t row = L.row_off32[d];
                for (int64_t i = doc_ptr[d]; i < doc_ptr[d + 1]; ++i) {
                    const uint32_t p = next[words[i]]++;
                    L.doc_map[i] = p;
                    L.tok_row[p] = row;
                    L.tok_crank[p] = ctmp[i];
                }
            }
        });
        if (on_final && !dev_scatter)
            on_final(pos_tile, pos, static_cast<uint64_t>(doc_ptr[d0]), static_cast<uint64_t>(doc_ptr[d1]));
    }
    if (on_final && !dev_scatter && tail_tokens > 0) on_final(static_cast<uint64_t>(T - tail_tokens), static_cast<uint64_t>(T), 0, 0);
    if (pos != static_cast<uint64_t>(T - tail_tokens)) return "internal: token layout does not cover the corpus";
    ctmp.release();
    tmark("layout: tiles (count, ranks, scatter)");
    tmark("layout: canonical ranks");
    // Tile sampler items: the (tile, word) runs in pieces of at most
    // chunk_tokens, tile by tile, heavy-first inside each tile.
    L.titems.clear();
    if (sampler == 2) {
        // tiles in parallel (threads take tiles in turn), then concatenated in tile order
        std::vector<std::vector<TileItem>> per(nt);
        std::atomic<int> next_tile{0};
        auto make = [&] {
            for (int b; (b = next_tile.fetch_add(1)) < nt;) {
                auto &it = per[b];
                for (int32_t w = 0; w < V; ++w) {
                    const int64_t n = tile_cnt[b][w];
                    if (n == 0) continue;
                    const int64_t pieces = (n + chunk_tokens - 1) / chunk_tokens;
                    const uint32_t pos = tseg[static_cast<size_t>(b) * V + w];
                    for (int64_t q = 0; q < pieces; ++q) {
                        const int64_t vb = n * q / pieces, ve = n * (q + 1) / pieces;
                        it.push_back(TileItem{static_cast<uint32_t>(w), pos + static_cast<uint32_t>(vb),
                                              static_cast<uint32_t>(ve - vb),
                                              tcrank[static_cast<size_t>(b) * V + w] + static_cast<uint32_t>(vb)});
                    }
                }
                std::stable_sort(it.begin(), it.end(), [](const TileItem &x, const TileItem &y) { return x.n > y.n; });
            }
        };
        {
            std::vector<std::thread> th;
            for (int t = 1; t < std::min(nthreads, nt); ++t) th.emplace_back(make);
            make();
            for (auto &x : th) x.join();
        }
        size_t total = 0;
        for (auto &it : per) total += it.size();
        if (total >= (uint64_t(1) << 32) - 1) return "too many tile sampler items";
        L.titems.reserve(total);
        for (auto &it : per) L.titems.insert(L.titems.end(), it.begin(), it.end());
    }

    tmark("layout: tile items");
    // Per-word runs (tile order) + sentinel; segment index of each word's first run.
    L.segs.clear();
    std::vector<uint64_t> wseg0(V + 1);
    for (int32_t w = 0; w < V; ++w) {
        wseg0[w] = L.segs.size();
        uint32_t acc = 0;
        for (int b = 0; b < nt; ++b) {
            uint32_t n = tile_cnt[b][w];
            if (n == 0) continue;
            L.segs.push_back(Seg{tseg[static_cast<size_t>(b) * V + w], acc});
            acc += n;
        }
        L.segs.push_back(Seg{0u, acc});
    }
    wseg0[V] = L.segs.size();
    if (L.segs.size() >= (uint64_t(1) << 32)) return "too many word runs";
    std::vector<uint32_t>().swap(tseg);
    auto seg_of = [&](int32_t w, uint32_t v) {
        uint64_t s = wseg0[w];
        while (L.segs[s + 1].vstart <= v && L.segs[s + 1].vstart < L.word_count[w]) ++s;
        return static_cast<uint32_t>(s);
    };

    // Sampling work items: word w's tokens in near-equal pieces of at most
    // chunk_tokens, each a virtual range spanning the word's runs; the
    // canonical index continues word w's run on this rank (cbase[w] + v).
    L.chunks.clear();
    L.zero_words.clear();
    if (sampler != 2) {  // sampler 0 only (the tile samplers use their own items)
        for (int32_t w = 0; w < V; ++w) {
            const int64_t n = L.word_count[w];
            const int64_t pieces = (n + chunk_tokens - 1) / chunk_tokens;
            if (pieces != 1) L.zero_words.push_back(w);
            if (n == 0) continue;
            for (int64_t q = 0; q < pieces; ++q) {
                const int64_t vb = n * q / pieces, ve = n * (q + 1) / pieces;
                SampleChunk c;
                c.word = static_cast<uint32_t>(w);
                c.vbegin = static_cast<uint32_t>(vb);
                c.count = static_cast<uint32_t>(ve - vb);
                c.seg0 = seg_of(w, static_cast<uint32_t>(vb));
                c.segN = static_cast<uint32_t>(wseg0[w + 1] - 1);
                c.pad = pieces > 1 ? 1u : 0u;  // bit 0: the word is split over chunks
                c.c_base = static_cast<uint64_t>(cbase[w]);
                L.chunks.push_back(c);
            }
        }
        std::stable_sort(L.chunks.begin(), L.chunks.end(),
                         [](const SampleChunk &a, const SampleChunk &b) { return a.count > b.count; });
    }

    tmark("layout: runs + sampler chunks");
    // Recount work items: per word, pieces of at most recount_tokens.
    L.rchunks.clear();
    L.split_words.clear();
    for (int32_t w = 0; w < V; ++w) {
        const int64_t n = L.word_count[w];
        const int64_t pieces = std::max<int64_t>(1, (n + recount_tokens - 1) / recount_tokens);
        if (pieces > 1) L.split_words.push_back(w);
        for (int64_t q = 0; q < pieces; ++q) {
            const int64_t vb = n * q / pieces, ve = n * (q + 1) / pieces;
            RecountChunk c;
            c.word = static_cast<uint32_t>(w) | (pieces > 1 ? 0x80000000u : 0u);
            c.vbegin = static_cast<uint32_t>(vb);
            c.vcount = static_cast<uint32_t>(ve - vb);
            c.seg0 = n ? seg_of(w, static_cast<uint32_t>(vb)) : static_cast<uint32_t>(wseg0[w]);
            c.segN = static_cast<uint32_t>(wseg0[w + 1] - 1);
            c.pad[0] = c.pad[1] = c.pad[2] = 0;
            L.rchunks.push_back(c);
        }
    }
    std::stable_sort(L.rchunks.begin(), L.rchunks.end(),
                     [](const RecountChunk &a, const RecountChunk &b) { return a.vcount > b.vcount; });
    tmark("layout: recount chunks");
    return "";
}

}  // namespace lda
