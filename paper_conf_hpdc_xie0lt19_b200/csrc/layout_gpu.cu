// a0 on the device: the doc-word map (L1297-1303) of the tile layout.
//
// The layout orders a rank's tokens tile by tile (document tiles), inside a
// tile by word, inside a word by document order; the tokens of "tail" words
// (too few per tile) form one run per word after the last tile.
// That order is a stable sort of the tokens by the key
//     tail word : ndt·V + w          (the tail tile)
//     otherwise : tile(d)·V + w
// so the word-major position of document-order token i is the rank of i in
// that sort, and doc_map[i] = position.  The host keeps the per-(tile, word)
// counts (work items, runs, canonical ranks); only the per-token scatter runs
// here: keys from the uploaded words, a stable LSD radix sort of (key, i)
// (8-bit digits: block histograms, a scan, a stable block-local scatter with
// warp-level match ranking), then the inversion.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>

#include "lda_internal.h"

namespace lda {
namespace {

constexpr int kRsThreads = 256;                  // 8 warps
constexpr int kRsWarpItems = 512;                // contiguous elements per warp
constexpr int kRsBlock = 8 * kRsWarpItems;       // 4096 elements per block
constexpr int kRadix = 256;
constexpr int kScanChunk = 4096;
constexpr unsigned kAll = 0xffffffffu;
static_assert(kRsThreads == kRadix, "rs_scatter_kernel: one thread per digit");

// keys may alias words (each thread reads words[i] before writing keys[i])
__global__ void layout_keys_kernel(const uint32_t *__restrict__ doc_ptr32, const int32_t *words,
                                   const uint8_t *__restrict__ tail, const uint32_t *__restrict__ tile_doc, int ndt,
                                   uint32_t V, int64_t D, uint32_t *keys, uint32_t *__restrict__ vals) {
    const int lane = threadIdx.x & 31;
    const int64_t nw = static_cast<int64_t>(gridDim.x) * (blockDim.x >> 5);
    for (int64_t d = static_cast<int64_t>(blockIdx.x) * (blockDim.x >> 5) + (threadIdx.x >> 5); d < D; d += nw) {
        // the document's tile: the last b with tile_doc[b] <= d
        int lo = 0, hi = ndt;  // tile_doc[0] = 0 <= d < tile_doc[ndt] = D
        while (hi - lo > 1) {
            const int mid = (lo + hi) >> 1;
            if (tile_doc[mid] <= static_cast<uint32_t>(d)) lo = mid;
            else hi = mid;
        }
        const uint32_t tbase = static_cast<uint32_t>(lo) * V, tailbase = static_cast<uint32_t>(ndt) * V;
        const uint32_t s = doc_ptr32[d], e = doc_ptr32[d + 1];
        for (uint32_t i = s + lane; i < e; i += 32) {
            const uint32_t w = static_cast<uint32_t>(words[i]);
            keys[i] = (tail[w] ? tailbase : tbase) + w;
            vals[i] = i;
        }
    }
}

__global__ void rs_hist_kernel(const uint32_t *__restrict__ keys, uint64_t n, int shift, uint32_t mask,
                               uint32_t nblocks, uint32_t *__restrict__ hist) {
    __shared__ uint32_t cnt[kRadix];
    for (int d = threadIdx.x; d < kRadix; d += blockDim.x) cnt[d] = 0u;
    __syncthreads();
    const uint64_t b0 = static_cast<uint64_t>(blockIdx.x) * kRsBlock;
    for (int r = threadIdx.x; r < kRsBlock; r += blockDim.x) {
        const uint64_t i = b0 + r;
        if (i < n) atomicAdd(&cnt[(keys[i] >> shift) & mask], 1u);
    }
    __syncthreads();
    for (int d = threadIdx.x; d < kRadix; d += blockDim.x) hist[static_cast<uint64_t>(d) * nblocks + blockIdx.x] = cnt[d];
}

// exclusive scan of a[0..L): chunk sums, a scan of the sums, the chunks
__global__ void scan_reduce_kernel(const uint32_t *__restrict__ a, uint64_t L, uint32_t *__restrict__ sums) {
    __shared__ uint32_t sh[32];
    const uint64_t c0 = static_cast<uint64_t>(blockIdx.x) * kScanChunk;
    uint32_t v = 0;
    for (int r = threadIdx.x; r < kScanChunk; r += blockDim.x)
        if (c0 + r < L) v += a[c0 + r];
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(kAll, v, o);
    if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = v;
    __syncthreads();
    if (threadIdx.x == 0) {
        uint32_t t = 0;
        for (int w = 0; w < static_cast<int>(blockDim.x >> 5); ++w) t += sh[w];
        sums[blockIdx.x] = t;
    }
}

__global__ void scan_sums_kernel(uint32_t *__restrict__ sums, uint32_t m) {
    // one block: exclusive scan of m sums, 1024 at a time
    __shared__ uint32_t sh[32];
    __shared__ uint32_t carry;
    if (threadIdx.x == 0) carry = 0;
    __syncthreads();
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    for (uint32_t b = 0; b < m; b += blockDim.x) {
        const uint32_t i = b + threadIdx.x;
        const uint32_t v = i < m ? sums[i] : 0u;
        uint32_t x = v;
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(kAll, x, o);
            if (lane >= o) x += y;
        }
        if (lane == 31) sh[warp] = x;
        __syncthreads();
        uint32_t off = carry;
        for (int w = 0; w < warp; ++w) off += sh[w];
        if (i < m) sums[i] = off + x - v;
        __syncthreads();
        if (threadIdx.x == blockDim.x - 1) carry = off + x;
        __syncthreads();
    }
}

__global__ void scan_chunks_kernel(uint32_t *__restrict__ a, uint64_t L, const uint32_t *__restrict__ sums) {
    // block = one chunk, 1024 threads x 4 entries
    __shared__ uint32_t sh[32];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint64_t c0 = static_cast<uint64_t>(blockIdx.x) * kScanChunk + 4 * threadIdx.x;
    uint32_t v[4], t = 0;
#pragma unroll
    for (int k = 0; k < 4; ++k) {
        v[k] = c0 + k < L ? a[c0 + k] : 0u;
        t += v[k];
    }
    uint32_t x = t;
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(kAll, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) sh[warp] = x;
    __syncthreads();
    uint32_t off = sums[blockIdx.x];
    for (int w = 0; w < warp; ++w) off += sh[w];
    off += x - t;
#pragma unroll
    for (int k = 0; k < 4; ++k) {
        if (c0 + k < L) a[c0 + k] = off;
        off += v[k];
    }
}

// stable scatter of one digit pass: warp w of block b owns elements
// [b·4096 + 512w, +512) and places them, in index order, after every element
// with a smaller digit and after the same digit's elements of earlier warps
// and blocks (hist: the scanned digit-major block histograms).  A lane holds
// its 16 elements in registers (all loads issued up front), ranks them within
// the warp with match_any once, and the block reorders its 4096 elements by
// digit in shared memory first, so that consecutive threads store
// consecutive addresses of a digit's run (coalesced) instead of 32 lanes
// storing into 32 different runs.
__global__ void __launch_bounds__(kRsThreads) rs_scatter_kernel(const uint32_t *__restrict__ kin,
                                                                const uint32_t *__restrict__ vin,
                                                                uint32_t *__restrict__ kout,
                                                                uint32_t *__restrict__ vout, uint64_t n, int shift,
                                                                uint32_t mask, uint32_t nblocks,
                                                                const uint32_t *__restrict__ hist) {
    constexpr int kIt = kRsWarpItems / 32;  // 16 elements per lane
    __shared__ uint32_t wcnt[8][kRadix];    // per-warp digit counts, then the warp's start in the block
    __shared__ uint32_t lstart[kRadix];     // block-local start of each digit's run
    __shared__ uint32_t gbase[kRadix];      // the block's global start of each digit's run
    __shared__ uint32_t wsum[8];
    __shared__ uint32_t sk[kRsBlock], sv[kRsBlock];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    for (int d = lane; d < kRadix; d += 32) wcnt[warp][d] = 0u;
    __syncwarp();
    const uint64_t b0 = static_cast<uint64_t>(blockIdx.x) * kRsBlock;
    const uint64_t w0 = b0 + static_cast<uint64_t>(warp) * kRsWarpItems;
    const unsigned lt = (1u << lane) - 1u;
    uint32_t k[kIt], v[kIt], off[kIt];
#pragma unroll
    for (int r = 0; r < kIt; ++r) {
        const uint64_t i = w0 + 32 * r + lane;
        k[r] = i < n ? kin[i] : 0u;
        v[r] = i < n ? vin[i] : 0u;
    }
    // the warp's digit counts; off = the element's rank among the warp's
    // elements of its digit
#pragma unroll
    for (int r = 0; r < kIt; ++r) {
        const uint64_t i = w0 + 32 * r + lane;
        const uint32_t d = i < n ? (k[r] >> shift) & mask : kRadix + lane;
        const unsigned peers = __match_any_sync(kAll, d);
        off[r] = 0u;
        if (i < n) off[r] = wcnt[warp][d] + __popc(peers & lt);
        __syncwarp();
        if (i < n && (peers & lt) == 0u) wcnt[warp][d] += __popc(peers);
        __syncwarp();
    }
    __syncthreads();
    // per digit (thread d): the warps' starts inside the digit's block run,
    // the run's length, then an exclusive scan of the lengths over digits
    uint32_t len = 0;
    {
        const int d = threadIdx.x;  // kRsThreads == kRadix
        for (int w = 0; w < 8; ++w) {
            const uint32_t c = wcnt[w][d];
            wcnt[w][d] = len;
            len += c;
        }
        gbase[d] = hist[static_cast<uint64_t>(d) * nblocks + blockIdx.x];
        uint32_t x = len;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(kAll, x, o);
            if (lane >= o) x += y;
        }
        if (lane == 31) wsum[warp] = x;
        __syncthreads();
        uint32_t pre = 0;
        for (int w = 0; w < warp; ++w) pre += wsum[w];
        lstart[d] = pre + x - len;
    }
    __syncthreads();
    // block-local placement in digit order
#pragma unroll
    for (int r = 0; r < kIt; ++r) {
        const uint64_t i = w0 + 32 * r + lane;
        if (i < n) {
            const uint32_t d = (k[r] >> shift) & mask;
            const uint32_t lp = lstart[d] + wcnt[warp][d] + off[r];
            sk[lp] = k[r];
            sv[lp] = v[r];
        }
    }
    __syncthreads();
    // coalesced stores: element t of the block's digit-ordered run
    const uint32_t nb = static_cast<uint32_t>(n - b0 < static_cast<uint64_t>(kRsBlock) ? n - b0 : kRsBlock);
    for (uint32_t t = threadIdx.x; t < nb; t += kRsThreads) {
        const uint32_t kk = sk[t];
        const uint32_t d = (kk >> shift) & mask;
        const uint32_t pos = gbase[d] + (t - lstart[d]);
        kout[pos] = kk;
        vout[pos] = sv[t];
    }
}

// doc_map[vals[p]] = p.  One thread per position and no grid-stride loop:
// blocks start in position order, so the scattered stores of the blocks in
// flight stay inside one document tile's part of doc_map (L2-resident; a
// grid-stride loop lets the blocks drift apart and the stores miss L2:
// 24.6 -> 9.7 ms at PubMed shape)
__global__ void invert_kernel(const uint32_t *__restrict__ vals, uint32_t *__restrict__ doc_map, uint64_t n) {
    const uint64_t p = static_cast<uint64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
    if (p < n) doc_map[vals[p]] = static_cast<uint32_t>(p);
}

}  // namespace

size_t radix_sort_temp_words(uint64_t n) {
    const uint64_t nblocks = (n + kRsBlock - 1) / kRsBlock;
    const uint64_t L = static_cast<uint64_t>(kRadix) * nblocks;
    return L + (L + kScanChunk - 1) / kScanChunk + 16;
}

int radix_sort_pairs(uint32_t *keys, uint32_t *vals, uint32_t *keys_tmp, uint32_t *vals_tmp, uint64_t n, int bits,
                     uint32_t *temp, void *stream, bool *result_in_tmp) {
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    *result_in_tmp = false;
    if (n == 0) return cudaSuccess;
    const uint32_t nblocks = static_cast<uint32_t>((n + kRsBlock - 1) / kRsBlock);
    const uint64_t L = static_cast<uint64_t>(kRadix) * nblocks;
    const uint32_t nchunks = static_cast<uint32_t>((L + kScanChunk - 1) / kScanChunk);
    uint32_t *hist = temp, *sums = temp + L;
    uint32_t *kin = keys, *vin = vals, *kout = keys_tmp, *vout = vals_tmp;
    for (int shift = 0; shift < std::max(bits, 1); shift += 8) {
        const int nb = std::min(8, bits - shift);
        const uint32_t mask = nb <= 0 ? 0u : (1u << nb) - 1u;
        rs_hist_kernel<<<nblocks, kRsThreads, 0, st>>>(kin, n, shift, mask, nblocks, hist);
        scan_reduce_kernel<<<nchunks, 1024, 0, st>>>(hist, L, sums);
        scan_sums_kernel<<<1, 1024, 0, st>>>(sums, nchunks);
        scan_chunks_kernel<<<nchunks, 1024, 0, st>>>(hist, L, sums);
        rs_scatter_kernel<<<nblocks, kRsThreads, 0, st>>>(kin, vin, kout, vout, n, shift, mask, nblocks, hist);
        std::swap(kin, kout);
        std::swap(vin, vout);
        *result_in_tmp = !*result_in_tmp;
    }
    return cudaGetLastError();
}

int launch_layout_keys(const uint32_t *doc_ptr32, const int32_t *words, const uint8_t *tail, const uint32_t *tile_doc,
                       int ndt, int32_t V, int64_t D, uint32_t *keys, uint32_t *vals, int num_sms, void *stream) {
    if (D > 0)
        layout_keys_kernel<<<num_sms * 8, 256, 0, static_cast<cudaStream_t>(stream)>>>(
            doc_ptr32, words, tail, tile_doc, ndt, static_cast<uint32_t>(V), D, keys, vals);
    return cudaGetLastError();
}

int launch_invert(const uint32_t *vals, uint32_t *doc_map, uint64_t n, void *stream) {
    if (n > 0)
        invert_kernel<<<static_cast<unsigned>((n + 255) / 256), 256, 0, static_cast<cudaStream_t>(stream)>>>(
            vals, doc_map, n);
    return cudaGetLastError();
}

}  // namespace lda

// Diagnostic (include/lda.h): the device radix sort on host arrays.
extern "C" int lda_debug_radix_sort(const uint32_t *keys, const uint32_t *vals, int64_t n, int32_t bits,
                                    uint32_t *out_keys, uint32_t *out_vals) {
    if (n < 0 || bits < 0 || bits > 32 || (n > 0 && (!keys || !vals || !out_keys || !out_vals))) return -1;
    if (n == 0) return 0;
    const size_t bytes = sizeof(uint32_t) * static_cast<size_t>(n);
    uint32_t *dk = nullptr, *dv = nullptr, *tk = nullptr, *tv = nullptr, *tmp = nullptr;
    cudaError_t e = cudaMalloc(&dk, bytes);
    if (e == cudaSuccess) e = cudaMalloc(&dv, bytes);
    if (e == cudaSuccess) e = cudaMalloc(&tk, bytes);
    if (e == cudaSuccess) e = cudaMalloc(&tv, bytes);
    if (e == cudaSuccess) e = cudaMalloc(&tmp, sizeof(uint32_t) * lda::radix_sort_temp_words(static_cast<uint64_t>(n)));
    if (e == cudaSuccess) e = cudaMemcpy(dk, keys, bytes, cudaMemcpyHostToDevice);
    if (e == cudaSuccess) e = cudaMemcpy(dv, vals, bytes, cudaMemcpyHostToDevice);
    bool in_tmp = false;
    if (e == cudaSuccess)
        e = static_cast<cudaError_t>(lda::radix_sort_pairs(dk, dv, tk, tv, static_cast<uint64_t>(n), bits, tmp,
                                                           nullptr, &in_tmp));
    if (e == cudaSuccess) e = cudaDeviceSynchronize();
    if (e == cudaSuccess) e = cudaMemcpy(out_keys, in_tmp ? tk : dk, bytes, cudaMemcpyDeviceToHost);
    if (e == cudaSuccess) e = cudaMemcpy(out_vals, in_tmp ? tv : dv, bytes, cudaMemcpyDeviceToHost);
    for (void *p : {static_cast<void *>(dk), static_cast<void *>(dv), static_cast<void *>(tk),
                    static_cast<void *>(tv), static_cast<void *>(tmp)})
        if (p) cudaFree(p);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return -4;  // LDA_ECUDA
    }
    return 0;
}
