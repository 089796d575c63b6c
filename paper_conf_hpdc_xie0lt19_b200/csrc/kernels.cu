// CUDA kernels of the LDA collapsed-Gibbs sweep, written for sm_100a (B200).
//
// Path per sweep t (§6):
//   prologue_kernel   invk[k] = 1/(n_k + Vβ)                (Eq. 1/8 denominator)
//   sweep_kernel      per word chunk: p*(k) = (n_wk+β)·invk[k] and the dense
//                     prefix of α·p* in shared memory (Eq. 8);
//                     per token: sparse doc row walk, S, one Philox uniform,
//                     x = U·(S+Q), group ballot search in the sparse prefix or a
//                     32-ary ballot search in the dense prefix (Eq. 6-7,
//                     Fig. 5, Alg. 2; L1019-1133)
//   recount_kernel    n_wk, n_k rebuilt from z by per-word segmented histograms
//                     (ϕ update, L1273-1285)
//   theta_kernel      per document: gather z through the doc-word map,
//                     histogram, ascending compaction into the θ row (θ
//                     update, L1287-1309; Eq. 5 invariant)
//   loglik kernels    fp64 lgamma reductions (Fig. 8; reading X11)
// No tensor cores: the path is a memory-bound gather/scan, not a contraction
// (Table 1, 0.19-0.33 flop/B, L555-563).
#include <cuda_runtime.h>

#include <cstdint>

#include "lda_internal.h"

namespace lda {

constexpr unsigned kFull = 0xffffffffu;
constexpr int kSweepThreads = 256;

// ---------------------------------------------------------------------------
// Philox4x32-10 (Salmon et al. SC'11), output word 0 only.  Counter
// (c lo, c hi, t, 0), key (seed lo, seed hi) (reading X9).
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint32_t philox_x0(uint64_t c, uint32_t t, uint32_t k0, uint32_t k1) {
    uint32_t c0 = static_cast<uint32_t>(c), c1 = static_cast<uint32_t>(c >> 32), c2 = t, c3 = 0u;
#pragma unroll
    for (int r = 0; r < 10; ++r) {
        const uint32_t hi0 = __umulhi(0xD2511F53u, c0), lo0 = 0xD2511F53u * c0;
        const uint32_t hi1 = __umulhi(0xCD9E8D57u, c2), lo1 = 0xCD9E8D57u * c2;
        c0 = hi1 ^ c1 ^ k0;
        c1 = lo1;
        c2 = hi0 ^ c3 ^ k1;
        c3 = lo0;
        k0 += 0x9E3779B9u;
        k1 += 0xBB67AE85u;
    }
    return c0;
}

__device__ __forceinline__ uint4 ld_nc_v4(const uint4 *p) {
    uint4 v;
    asm volatile("ld.global.nc.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
                 : "l"(p));
    return v;
}

// ---------------------------------------------------------------------------
// a1: random initial assignment (L377-379; X10): z = (x0·K) >> 32, t = 0.
// ---------------------------------------------------------------------------
__global__ void init_kernel(const SampleChunk *__restrict__ chunks, int64_t n_chunks,
                            uint16_t *__restrict__ z, uint32_t K, uint32_t k0, uint32_t k1) {
    for (int64_t ci = blockIdx.x; ci < n_chunks; ci += gridDim.x) {
        const SampleChunk ch = chunks[ci];
        for (uint32_t j = threadIdx.x; j < ch.count; j += blockDim.x) {
            const uint32_t x0 = philox_x0(ch.c_base + j, 0u, k0, k1);
            z[ch.begin + j] = static_cast<uint16_t>((static_cast<uint64_t>(x0) * K) >> 32);
        }
    }
}

// ---------------------------------------------------------------------------
// a2: sweep prologue, invk[k] = 1 / (n_k + Vβ)  (fp64).
// ---------------------------------------------------------------------------
__global__ void prologue_kernel(const int32_t *__restrict__ nk, int K, double Vbeta,
                                double *__restrict__ invk) {
    for (int k = blockIdx.x * blockDim.x + threadIdx.x; k < K; k += gridDim.x * blockDim.x)
        invk[k] = 1.0 / (static_cast<double>(nk[k]) + Vbeta);
}

// ---------------------------------------------------------------------------
// a3 + a4: the sampling kernel.
// ---------------------------------------------------------------------------
struct SweepArgs {
    const SampleChunk *chunks;
    int64_t n_chunks;
    const uint32_t *tok_row;
    uint16_t *z;
    const uint4 *rows;
    const int32_t *nwk;
    const int32_t *nk;
    const double *invk;
    uint32_t *counter;
    double *gscratch;  // non-null when the K-length arrays do not fit in smem
    int K;
    int top_step;
    double alpha, beta, Vbeta;
    uint32_t t, k0, k1;
};

// One token, drawn by a group of GS lanes (GS | 32).  Returns the new topic
// on every lane of the group.
//   row layout: word 0 = nnz, words 1..nnz = (topic << 16 | count), topics
//   ascending (X7).  Lane q of the group owns words 4q..4q+3 of each 4·GS-word
//   slice; its masses are count·p*(topic) (p1 of Eq. 6 via Eq. 8).
// Bins: [sparse entries in row order] ++ [dense α·p*(k), k = 0..K-1] (X4-X6).
template <int GS, bool EXCL>
__device__ __forceinline__ int draw_token(const SweepArgs &a, const double *__restrict__ pstar,
                                          const double *__restrict__ P, double Q,
                                          const int32_t *__restrict__ nwk_row, uint32_t trow,
                                          uint32_t x0, int zo, unsigned gmask, int q, int gbase) {
    const uint4 *r = a.rows + trow;
    uint4 v = ld_nc_v4(r + q);
    const uint32_t len = __shfl_sync(gmask, v.x, gbase);
    const uint32_t nwords = len + 1;
    const int iters = static_cast<int>((nwords + 4 * GS - 1) / (4 * GS));

    // exclude_self (X2 optional variant): the token's own topic zo loses one
    // count in n_dk, n_wk and n_k.
    double po_new = 0.0, delta = 0.0;
    if (EXCL) {
        po_new = (static_cast<double>(nwk_row[zo] - 1) + a.beta) /
                 (static_cast<double>(a.nk[zo] - 1) + a.Vbeta);
        delta = a.alpha * po_new - a.alpha * pstar[zo];
    }

    double c0 = 0, c1 = 0, c2 = 0, c3 = 0;
    uint32_t e0 = 0, e1 = 0, e2 = 0, e3 = 0;
    uint32_t wb = 0;  // word index of this lane's first word in the slice

    // computes c0..c3 for slice `it` from v; returns the slice's group total
    auto slice = [&](int it, double carry) -> double {
        wb = static_cast<uint32_t>(it * 4 * GS + 4 * q);
        e0 = v.x; e1 = v.y; e2 = v.z; e3 = v.w;
        double m0 = 0, m1 = 0, m2 = 0, m3 = 0;
#define LDA_MASS(mi, ei, off)                                                              \
    if (wb + off >= 1 && wb + off <= len) {                                                \
        const uint32_t tp = ei >> 16, cn = ei & 0xFFFFu;                                   \
        mi = (EXCL && static_cast<int>(tp) == zo) ? static_cast<double>(cn - 1) * po_new   \
                                                  : static_cast<double>(cn) * pstar[tp];   \
    }
        LDA_MASS(m0, e0, 0)
        LDA_MASS(m1, e1, 1)
        LDA_MASS(m2, e2, 2)
        LDA_MASS(m3, e3, 3)
#undef LDA_MASS
        const double l0 = m0, l1 = l0 + m1, l2 = l1 + m2, l3 = l2 + m3;
        double incl = l3;
#pragma unroll
        for (int o = 1; o < GS; o <<= 1) {
            const double y = __shfl_up_sync(gmask, incl, o, GS);
            if (q >= o) incl += y;
        }
        double ex = __shfl_up_sync(gmask, incl, 1, GS);
        if (q == 0) ex = 0.0;
        const double base = carry + ex;
        c0 = base + l0;
        c1 = base + l1;
        c2 = base + l2;
        c3 = base + l3;
        return __shfl_sync(gmask, incl, GS - 1, GS);
    };

    // pass 1: S = inclusive prefix at the last sparse entry (word `len`)
    double carry = 0.0, S = 0.0;
    for (int it = 0; it < iters; ++it) {
        if (it > 0) {
            const uint32_t w0 = static_cast<uint32_t>(it * 4 * GS + 4 * q);
            v = (w0 < nwords) ? ld_nc_v4(r + it * GS + q) : make_uint4(0u, 0u, 0u, 0u);
        }
        const double tot = slice(it, carry);
        if (it == iters - 1 && len > 0) {
            const uint32_t rel = len - static_cast<uint32_t>(it * 4 * GS);
            const int src = gbase + static_cast<int>(rel >> 2);
            const uint32_t i = rel & 3u;
            const double mine = i == 0 ? c0 : (i == 1 ? c1 : (i == 2 ? c2 : c3));
            S = __shfl_sync(gmask, mine, src);
        }
        carry = carry + tot;
    }

    const double U = static_cast<double>(x0) * 2.3283064365386962890625e-10;  // x0 · 2^-32
    const double x = U * (S + (EXCL ? Q + delta : Q));

    if (x < S) {
        // sparse bucket (p1): first entry with C > x.  For rows longer than
        // one slice, recompute each slice bit-identically to pass 1.
        double carry2 = 0.0;
        for (int it = 0; it < iters; ++it) {
            double tot = 0.0;
            if (iters > 1) {
                const uint32_t w0 = static_cast<uint32_t>(it * 4 * GS + 4 * q);
                v = (w0 < nwords) ? ld_nc_v4(r + it * GS + q) : make_uint4(0u, 0u, 0u, 0u);
                tot = slice(it, carry2);
            }
            const bool f0 = wb + 0 >= 1 && wb + 0 <= len && c0 > x;
            const bool f1 = wb + 1 >= 1 && wb + 1 <= len && c1 > x;
            const bool f2 = wb + 2 >= 1 && wb + 2 <= len && c2 > x;
            const bool f3 = wb + 3 >= 1 && wb + 3 <= len && c3 > x;
            const unsigned bal = __ballot_sync(gmask, f0 || f1 || f2 || f3) & gmask;
            if (bal) {
                const uint32_t e = f0 ? e0 : (f1 ? e1 : (f2 ? e2 : e3));
                return static_cast<int>(__shfl_sync(gmask, e, __ffs(bal) - 1) >> 16);
            }
            carry2 = carry2 + tot;
        }
        return a.K - 1;  // unreachable: the entry at word `len` has C == S > x
    }

    // dense bucket (p2): first k with S + P[k] (+Δ for k >= zo) > x, by a
    // 32-ary search whose candidates are split over the group's lanes
    // (the index tree of Fig. 5 / Fig. 6).
    constexpr int PER = 32 / GS;
    int base = 0, step = a.top_step;
    for (;;) {
        int first = 32;
#pragma unroll
        for (int i = 0; i < PER; ++i) {
            const int j = q * PER + i;
            int idx = base + (j + 1) * step - 1;
            if (idx > a.K - 1) idx = a.K - 1;
            double pk = P[idx];
            if (EXCL && idx >= zo) pk += delta;
            if (first == 32 && S + pk > x) first = j;
        }
        const unsigned bal = __ballot_sync(gmask, first < 32) & gmask;
        int js;
        if (bal) {
            js = __shfl_sync(gmask, first, __ffs(bal) - 1);
        } else {
            if (step == a.top_step) return a.K - 1;  // x >= total (rounding), X6 fallback
            js = 31;
        }
        if (step == 1) return min(base + js, a.K - 1);
        base += js * step;
        step >>= 5;
    }
}

template <int GS, bool EXCL>
__global__ void __launch_bounds__(kSweepThreads) sweep_kernel(SweepArgs a) {
    extern __shared__ double smem_d[];
    __shared__ int s_ci;
    __shared__ double s_wtot[kSweepThreads / 32];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    constexpr int NG = 32 / GS;
    const int g = lane / GS, q = lane % GS, gbase = g * GS;
    const unsigned gmask = (GS == 32) ? kFull : (((1u << GS) - 1u) << gbase);
    const int K = a.K;
    double *pstar = a.gscratch ? a.gscratch + static_cast<size_t>(blockIdx.x) * 2 * K : smem_d;
    double *P = pstar + K;
    const int E = (K + kSweepThreads - 1) / kSweepThreads;
    int cur_word = -1;

    for (;;) {
        if (tid == 0) s_ci = static_cast<int>(atomicAdd(a.counter, 1u));
        __syncthreads();
        const int ci = s_ci;
        if (ci >= a.n_chunks) break;
        const SampleChunk ch = a.chunks[ci];
        const int32_t *nwk_row = a.nwk + static_cast<size_t>(ch.word) * K;

        if (static_cast<int>(ch.word) != cur_word) {
            // p*(k) and the inclusive prefix of α·p*(k) for this word (Eq. 8)
            const int kb = tid * E;
            double run = 0.0;
            for (int e = 0; e < E; ++e) {
                const int k = kb + e;
                if (k < K) {
                    const double ps = (static_cast<double>(__ldg(nwk_row + k)) + a.beta) * __ldg(a.invk + k);
                    pstar[k] = ps;
                    run = run + a.alpha * ps;
                    P[k] = run;
                }
            }
            double incl = run;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const double y = __shfl_up_sync(kFull, incl, o);
                if (lane >= o) incl += y;
            }
            double lex = __shfl_up_sync(kFull, incl, 1);
            if (lane == 0) lex = 0.0;
            if (lane == 31) s_wtot[warp] = incl;
            __syncthreads();
            double off = 0.0;
            for (int i = 0; i < warp; ++i) off += s_wtot[i];
            off = off + lex;
            for (int e = 0; e < E; ++e) {
                const int k = kb + e;
                if (k < K) P[k] = off + P[k];
            }
            __syncthreads();
            cur_word = static_cast<int>(ch.word);
        }
        const double Q = P[K - 1];

        for (uint32_t b0 = static_cast<uint32_t>(warp) * 32; b0 < ch.count; b0 += kSweepThreads) {
            const uint32_t jj = b0 + lane;
            const bool valid = jj < ch.count;
            const uint32_t p = ch.begin + jj;
            const uint32_t row = valid ? __ldg(a.tok_row + p) : 0u;
            const uint32_t x0 = philox_x0(ch.c_base + jj, a.t, a.k0, a.k1);
            const int zo = (EXCL && valid) ? static_cast<int>(a.z[p]) : 0;
            int myz = 0;
#pragma unroll 1
            for (int r = 0; r < GS; ++r) {
                const int j = r * NG + g;
                const uint32_t trow = __shfl_sync(kFull, row, j);
                const uint32_t tx0 = __shfl_sync(kFull, x0, j);
                const int tzo = __shfl_sync(kFull, zo, j);
                int zn = 0;
                if (b0 + static_cast<uint32_t>(j) < ch.count)
                    zn = draw_token<GS, EXCL>(a, pstar, P, Q, nwk_row, trow, tx0, tzo, gmask, q, gbase);
                const int got = __shfl_sync(kFull, zn, (lane % NG) * GS);
                if (r == lane / NG) myz = got;
            }
            if (valid) a.z[p] = static_cast<uint16_t>(myz);
        }
        __syncthreads();
    }
}

// ---------------------------------------------------------------------------
// a4 epilogue (separate kernel): n_wk / n_k recount from z.
// ---------------------------------------------------------------------------
__global__ void zero_rows_kernel(const int32_t *__restrict__ words, int64_t n, int32_t *__restrict__ nwk,
                                 int K) {
    for (int64_t i = blockIdx.x; i < n; i += gridDim.x) {
        int32_t *row = nwk + static_cast<size_t>(words[i]) * K;
        for (int k = threadIdx.x; k < K; k += blockDim.x) row[k] = 0;
    }
}

__global__ void recount_kernel(const RecountChunk *__restrict__ rc, int64_t n_rc,
                               const uint32_t *__restrict__ tseg, int ntiles, int V, int K,
                               const uint16_t *__restrict__ z, int32_t *__restrict__ nwk,
                               int32_t *__restrict__ nk, uint32_t *__restrict__ counter) {
    extern __shared__ int smem_i[];
    int *hist = smem_i, *nkp = smem_i + K;
    __shared__ int s_ci;
    for (int k = threadIdx.x; k < 2 * K; k += blockDim.x) smem_i[k] = 0;
    __syncthreads();
    for (;;) {
        if (threadIdx.x == 0) s_ci = static_cast<int>(atomicAdd(counter, 1u));
        __syncthreads();
        const int ci = s_ci;
        if (ci >= n_rc) break;
        const RecountChunk c = rc[ci];
        const uint32_t vb = c.vbegin, ve = c.vbegin + c.vcount;
        uint32_t acc = 0;
        for (int b = 0; b < ntiles && acc < ve; ++b) {
            const size_t key = static_cast<size_t>(b) * V + c.word;
            const uint32_t s = tseg[key], n = tseg[key + 1] - s;
            const uint32_t lo = max(vb, acc), hi = min(ve, acc + n);
            for (uint32_t vv = lo + threadIdx.x; vv < hi; vv += blockDim.x)
                atomicAdd(&hist[z[s + (vv - acc)]], 1);
            acc += n;
        }
        __syncthreads();
        int32_t *row = nwk + static_cast<size_t>(c.word) * K;
        for (int k = threadIdx.x; k < K; k += blockDim.x) {
            const int h = hist[k];
            if (c.split) {
                if (h) atomicAdd(row + k, h);
            } else {
                row[k] = h;
            }
            nkp[k] += h;
            hist[k] = 0;
        }
        __syncthreads();
    }
    for (int k = threadIdx.x; k < K; k += blockDim.x)
        if (nkp[k]) atomicAdd(nk + k, nkp[k]);
}

// ---------------------------------------------------------------------------
// a5: θ rebuild.  One warp per document: gather z through the doc-word map,
// count topics in a per-warp shared histogram + bitmap, then write the row
// as ascending (topic << 16 | count) entries with a popc scan over the bitmap.
// O(L_d + K/32) per document instead of the paper's dense O(K) row.
// ---------------------------------------------------------------------------
__global__ void theta_kernel(const uint32_t *__restrict__ doc_ptr32, const uint32_t *__restrict__ row_off16,
                             const uint32_t *__restrict__ doc_map, const uint16_t *__restrict__ z,
                             uint32_t *__restrict__ rows, int64_t D, int K,
                             unsigned long long *__restrict__ stat) {
    extern __shared__ uint32_t smem_u[];
    const int Kw = (K + 31) >> 5;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, wpb = blockDim.x >> 5;
    uint32_t *cnt = smem_u + static_cast<size_t>(warp) * (K + Kw);
    uint32_t *bits = cnt + K;
    for (int k = lane; k < K + Kw; k += 32) cnt[k] = 0u;
    __syncwarp();
    unsigned long long s_lnnz = 0, s_nnz = 0;
    const int64_t nw = static_cast<int64_t>(gridDim.x) * wpb;
    for (int64_t d = static_cast<int64_t>(blockIdx.x) * wpb + warp; d < D; d += nw) {
        const uint32_t s = doc_ptr32[d], e = doc_ptr32[d + 1];
        for (uint32_t i = s + lane; i < e; i += 32) {
            const uint32_t k = z[doc_map[i]];
            atomicAdd(&cnt[k], 1u);
            atomicOr(&bits[k >> 5], 1u << (k & 31));
        }
        __syncwarp();
        uint32_t *row = rows + static_cast<size_t>(row_off16[d]) * 4;
        uint32_t base = 0;
        for (int qb = 0; qb < Kw; qb += 32) {
            const int qq = qb + lane;
            uint32_t bw = qq < Kw ? bits[qq] : 0u;
            const uint32_t pc = __popc(bw);
            uint32_t incl = pc;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t y = __shfl_up_sync(kFull, incl, o);
                if (lane >= o) incl += y;
            }
            uint32_t pos = base + incl - pc;
            while (bw) {
                const int b = __ffs(bw) - 1;
                bw &= bw - 1;
                const uint32_t k = static_cast<uint32_t>(qq) * 32 + b;
                row[1 + pos++] = (k << 16) | cnt[k];
                cnt[k] = 0u;
            }
            if (qq < Kw) bits[qq] = 0u;
            base += __shfl_sync(kFull, incl, 31);
        }
        if (lane == 0) {
            row[0] = base;
            s_nnz += base;
            s_lnnz += static_cast<unsigned long long>(e - s) * base;
        }
        __syncwarp();
    }
    if (lane == 0) {
        atomicAdd(stat + 0, s_lnnz);
        atomicAdd(stat + 1, s_nnz);
    }
}

// ---------------------------------------------------------------------------
// Log-likelihood (X11), deterministic two-stage fp64 reductions.
// ---------------------------------------------------------------------------
__device__ double block_sum(double v, double *sh) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_down_sync(kFull, v, o);
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    if (lane == 0) sh[warp] = v;
    __syncthreads();
    double t = 0.0;
    if (threadIdx.x == 0)
        for (int i = 0; i < (int)(blockDim.x >> 5); ++i) t += sh[i];
    __syncthreads();
    return t;
}

__global__ void ll_word_kernel(const int32_t *__restrict__ nwk, int64_t n, double beta, double lgb,
                               double *__restrict__ part) {
    __shared__ double sh[32];
    double s = 0.0;
    for (int64_t i = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x; i < n;
         i += static_cast<int64_t>(gridDim.x) * blockDim.x) {
        const int v = nwk[i];
        if (v) s += lgamma(static_cast<double>(v) + beta) - lgb;
    }
    const double t = block_sum(s, sh);
    if (threadIdx.x == 0) part[blockIdx.x] = t;
}

__global__ void ll_doc_kernel(const uint32_t *__restrict__ doc_ptr32, const uint32_t *__restrict__ row_off16,
                              const uint32_t *__restrict__ rows, int64_t D, double alpha, double lga,
                              double Kalpha, double lgKa, double *__restrict__ part) {
    __shared__ double sh[32];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, wpb = blockDim.x >> 5;
    double s = 0.0;
    const int64_t nw = static_cast<int64_t>(gridDim.x) * wpb;
    for (int64_t d = static_cast<int64_t>(blockIdx.x) * wpb + warp; d < D; d += nw) {
        const uint32_t *row = rows + static_cast<size_t>(row_off16[d]) * 4;
        const uint32_t nnz = row[0];
        if (lane == 0) s += lgKa - lgamma(static_cast<double>(doc_ptr32[d + 1] - doc_ptr32[d]) + Kalpha);
        for (uint32_t j = lane; j < nnz; j += 32)
            s += lgamma(static_cast<double>(row[1 + j] & 0xFFFFu) + alpha) - lga;
    }
    const double t = block_sum(s, sh);
    if (threadIdx.x == 0) part[blockIdx.x] = t;
}

__global__ void ll_final_kernel(const double *__restrict__ part_w, int nw, const double *__restrict__ part_d,
                                int nd, const int32_t *__restrict__ nk, int K, double Vbeta,
                                double lgVb, int word_part, double *__restrict__ out) {
    __shared__ double sh[32];
    double w = 0.0, d = 0.0;
    if (word_part) {
        for (int i = threadIdx.x; i < nw; i += blockDim.x) w += part_w[i];
        for (int k = threadIdx.x; k < K; k += blockDim.x)
            w += lgVb - lgamma(static_cast<double>(nk[k]) + Vbeta);
    }
    for (int i = threadIdx.x; i < nd; i += blockDim.x) d += part_d[i];
    const double tw = block_sum(w, sh);
    const double td = block_sum(d, sh);
    if (threadIdx.x == 0) {
        out[0] = tw;
        out[1] = td;
    }
}

// ---------------------------------------------------------------------------
// Launchers
// ---------------------------------------------------------------------------
static constexpr int kGS = 8;  // lanes per token in the sampler

static int top_step_for(int K) {
    int step = 1;
    while (static_cast<int64_t>(step) * 32 < K) step *= 32;
    return step;
}

int configure_kernels(DevState &s) {
    cudaError_t e;
    int dev = 0;
    if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
    if ((e = cudaDeviceGetAttribute(&s.num_sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess) return e;
    int max_optin = 0;
    if ((e = cudaDeviceGetAttribute(&max_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev)) != cudaSuccess)
        return e;
    // sampler
    size_t want = static_cast<size_t>(16) * s.K;
    s.sweep_smem = (want + 2048 <= static_cast<size_t>(max_optin)) ? want : 0;
    const void *fns[2] = {reinterpret_cast<const void *>(&sweep_kernel<kGS, false>),
                          reinterpret_cast<const void *>(&sweep_kernel<kGS, true>)};
    int bps = 1;
    for (int i = 0; i < 2; ++i) {
        if ((e = cudaFuncSetAttribute(fns[i], cudaFuncAttributeMaxDynamicSharedMemorySize,
                                      static_cast<int>(s.sweep_smem))) != cudaSuccess)
            return e;
    }
    if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, fns[s.exclude_self ? 1 : 0], kSweepThreads,
                                                           s.sweep_smem)) != cudaSuccess)
        return e;
    s.sweep_grid = s.num_sms * (bps > 0 ? bps : 1);
    // recount
    if ((e = cudaFuncSetAttribute(reinterpret_cast<const void *>(&recount_kernel),
                                  cudaFuncAttributeMaxDynamicSharedMemorySize, 8 * s.K)) != cudaSuccess)
        return e;
    // theta: as many warps per block (<= 8) as fit
    size_t per_warp = static_cast<size_t>(4) * (s.K + (s.K + 31) / 32);
    int wpb = static_cast<int>(std::min<size_t>(8, (static_cast<size_t>(max_optin) - 1024) / per_warp));
    if (wpb < 1) return cudaErrorInvalidValue;
    s.theta_block = 32 * wpb;
    s.theta_smem = per_warp * wpb;
    if ((e = cudaFuncSetAttribute(reinterpret_cast<const void *>(&theta_kernel),
                                  cudaFuncAttributeMaxDynamicSharedMemorySize,
                                  static_cast<int>(s.theta_smem))) != cudaSuccess)
        return e;
    int tb = 1;
    if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&tb, reinterpret_cast<const void *>(&theta_kernel),
                                                           s.theta_block, s.theta_smem)) != cudaSuccess)
        return e;
    s.theta_grid = s.num_sms * (tb > 0 ? tb : 1);
    s.ll_blocks = 2 * s.num_sms;
    return cudaSuccess;
}

int launch_init(const DevState &s, void *stream) {
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    const int grid = static_cast<int>(std::min<int64_t>(s.n_chunks > 0 ? s.n_chunks : 1, 65535));
    init_kernel<<<grid, 256, 0, st>>>(s.chunks, s.n_chunks, s.tok_z, static_cast<uint32_t>(s.K),
                                      static_cast<uint32_t>(s.seed), static_cast<uint32_t>(s.seed >> 32));
    return cudaGetLastError();
}

int launch_recount(const DevState &s, void *stream, int *launches) {
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    cudaError_t e;
    int32_t *nk = s.nwk + static_cast<size_t>(s.V) * s.K;
    if ((e = cudaMemsetAsync(nk, 0, sizeof(int32_t) * s.K, st)) != cudaSuccess) return e;
    if ((e = cudaMemsetAsync(s.counter + 1, 0, sizeof(uint32_t), st)) != cudaSuccess) return e;
    if (s.n_split > 0) {
        zero_rows_kernel<<<static_cast<int>(std::min<int64_t>(s.n_split, 65535)), 256, 0, st>>>(
            s.split_words, s.n_split, s.nwk, s.K);
        ++*launches;
    }
    recount_kernel<<<s.sweep_grid > 0 ? s.num_sms * 4 : 1, 256, 8 * s.K, st>>>(
        s.rchunks, s.n_rchunks, s.tseg, s.ntiles, s.V, s.K, s.tok_z, s.nwk, nk, s.counter + 1);
    ++*launches;
    return cudaGetLastError();
}

int launch_theta(const DevState &s, unsigned long long *stat_out, void *stream, int *launches) {
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    cudaError_t e;
    if ((e = cudaMemsetAsync(stat_out, 0, 2 * sizeof(unsigned long long), st)) != cudaSuccess) return e;
    theta_kernel<<<s.theta_grid, s.theta_block, s.theta_smem, st>>>(s.doc_ptr32, s.row_off16, s.doc_map,
                                                                     s.tok_z, s.rows, s.D, s.K, stat_out);
    ++*launches;
    return cudaGetLastError();
}

int launch_sweep(const DevState &s, uint32_t t, void *stream, int *launches) {
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    cudaError_t e;
    const double Vbeta = static_cast<double>(s.V) * s.beta;
    const int32_t *nk = s.nwk + static_cast<size_t>(s.V) * s.K;
    prologue_kernel<<<(s.K + 255) / 256, 256, 0, st>>>(nk, s.K, Vbeta, s.invk);
    ++*launches;
    if ((e = cudaMemsetAsync(s.counter, 0, sizeof(uint32_t), st)) != cudaSuccess) return e;
    SweepArgs a;
    a.chunks = s.chunks;
    a.n_chunks = s.n_chunks;
    a.tok_row = s.tok_row;
    a.z = s.tok_z;
    a.rows = reinterpret_cast<const uint4 *>(s.rows);
    a.nwk = s.nwk;
    a.nk = nk;
    a.invk = s.invk;
    a.counter = s.counter;
    a.gscratch = s.sweep_smem ? nullptr : s.sweep_scratch;  // large-K fallback
    a.K = s.K;
    a.top_step = top_step_for(s.K);
    a.alpha = s.alpha;
    a.beta = s.beta;
    a.Vbeta = Vbeta;
    a.t = t;
    a.k0 = static_cast<uint32_t>(s.seed);
    a.k1 = static_cast<uint32_t>(s.seed >> 32);
    if (s.exclude_self)
        sweep_kernel<kGS, true><<<s.sweep_grid, kSweepThreads, s.sweep_smem, st>>>(a);
    else
        sweep_kernel<kGS, false><<<s.sweep_grid, kSweepThreads, s.sweep_smem, st>>>(a);
    ++*launches;
    return cudaGetLastError();
}

int launch_loglik(const DevState &s, bool word_part, void *stream, int *launches) {
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    const double Vbeta = static_cast<double>(s.V) * s.beta, Kalpha = static_cast<double>(s.K) * s.alpha;
    double *pw = s.ll_part, *pd = s.ll_part + s.ll_blocks;
    int nw = 0;
    if (word_part) {
        ll_word_kernel<<<s.ll_blocks, 256, 0, st>>>(s.nwk, static_cast<int64_t>(s.V) * s.K, s.beta,
                                                    lgamma(s.beta), pw);
        nw = s.ll_blocks;
        ++*launches;
    }
    ll_doc_kernel<<<s.ll_blocks, 256, 0, st>>>(s.doc_ptr32, s.row_off16, s.rows, s.D, s.alpha, lgamma(s.alpha),
                                               Kalpha, lgamma(Kalpha), pd);
    ++*launches;
    ll_final_kernel<<<1, 256, 0, st>>>(pw, nw, pd, s.ll_blocks, s.nwk + static_cast<size_t>(s.V) * s.K, s.K,
                                       Vbeta, lgamma(Vbeta), word_part ? 1 : 0, s.ll_out);
    ++*launches;
    return cudaGetLastError();
}

}  // namespace lda
