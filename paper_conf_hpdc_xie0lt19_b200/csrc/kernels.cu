// CUDA kernels of the LDA collapsed-Gibbs sweep, written for sm_100a (B200).
//
// Path per sweep t (§6):
//   prologue_kernel   denom[k] = n_k + Vβ                    (Eq. 1/8 denominator)
//   sweep_kernel      per word chunk: p*(k) = (n_wk+β)/denom[k] and the dense
//                     prefix of α·p* in shared memory (Eq. 8);
//                     per token (one sampler per lane): sparse doc row walk,
//                     S, one Philox uniform, x = U·(S+Q), rescan of the sparse
//                     prefix or binary search of the dense prefix (Eq. 6-7,
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

#include <algorithm>
#include <cstdint>
#include <cstring>

#include "lda_internal.h"

namespace lda {

constexpr unsigned kFull = 0xffffffffu;
// θ row entry: topic << kTS | count (count < 2^16 in bits 0-15, bits 16-17
// zero), so that e >> 16 is the byte offset 4·topic of the topic in an fp32
// table.  K <= 16384 (14 topic bits).  Wide entries for 16384 < K <= 65536
// (u16 topic ids, L1239-1243): topic << kTSWide | count (sampler 0 only).
constexpr int kTS = 18;
constexpr int kTSWide = 16;
__host__ __device__ constexpr int entry_shift(int K) { return K > 16384 ? kTSWide : kTS; }
constexpr int kSweepThreads = 256;
constexpr int kMaxBlk = 16;  // block-end prefixes kept per token for the sparse rescan
#ifndef LDA_RING
#define LDA_RING 3
#endif
#ifndef LDA_FUSE
#define LDA_FUSE 1
#endif
#ifndef LDA_SWEEP_MINB
#define LDA_SWEEP_MINB 3
#endif
constexpr int kRing = LDA_RING;  // 32-byte row blocks in flight per sampler lane

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

// One 32-byte θ row block per lane: a single 256-bit load (sm_100 LDG.256).
struct Blk8 {
    uint32_t w[8];
};
__device__ __forceinline__ Blk8 ld_nc_v8(const uint32_t *p) {
    Blk8 b;
    asm volatile("ld.global.nc.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(b.w[0]), "=r"(b.w[1]), "=r"(b.w[2]), "=r"(b.w[3]), "=r"(b.w[4]), "=r"(b.w[5]),
                   "=r"(b.w[6]), "=r"(b.w[7])
                 : "l"(p));
    return b;
}

__device__ __forceinline__ uint4 ld_nc_v4(const uint4 *p) {
    uint4 v;
    asm volatile("ld.global.nc.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
                 : "l"(p));
    return v;
}

// L2 residency hints of the tile samplers (createpolicy + .L2::cache_hint):
// θ rows evict_last, the once-per-tile streams (tok_row, the per-item word
// tables) evict_first.  Measured on B200 at PubMed shape: 2.5 % SLOWER
// (policy registers at the 128-register limit; the kernel is bound by
// issue and load latency, not by DRAM bandwidth) -- off by default.
#ifndef LDA_L2HINT
#define LDA_L2HINT 0
#endif
__device__ __forceinline__ uint64_t pol_evict_last() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint64_t pol_evict_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
// a θ row line block (kept in L2)
__device__ __forceinline__ Blk8 ld_row_v8(const uint32_t *p) {
#if LDA_L2HINT
    Blk8 b;
    asm volatile("ld.global.nc.L2::cache_hint.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8], %9;"
                 : "=r"(b.w[0]), "=r"(b.w[1]), "=r"(b.w[2]), "=r"(b.w[3]), "=r"(b.w[4]), "=r"(b.w[5]),
                   "=r"(b.w[6]), "=r"(b.w[7])
                 : "l"(p), "l"(pol_evict_last()));
    return b;
#else
    return ld_nc_v8(p);
#endif
}
// a θ row header word (kept in L2)
__device__ __forceinline__ uint32_t ld_row_u32(const uint32_t *p) {
#if LDA_L2HINT
    uint32_t v;
    asm volatile("ld.global.nc.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol_evict_last()));
    return v;
#else
    return __ldg(p);
#endif
}
// a streamed word (tok_row: read once per sweep)
__device__ __forceinline__ uint32_t ld_stream_u32(const uint32_t *p) {
#if LDA_L2HINT
    uint32_t v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.u32 %0, [%1], %2;"
                 : "=r"(v)
                 : "l"(p), "l"(pol_evict_first()));
    return v;
#else
    return __ldg(p);
#endif
}

// Bring the 32-byte sector at p into L2 (no register, no scoreboard).
__device__ __forceinline__ void prefetch_l2(const void *p) {
    asm volatile("prefetch.global.L2 [%0];" ::"l"(p));
}

// Bring [p, p + bytes) into L2 without a register or scoreboard slot (one
// bulk-prefetch instruction per θ row; bytes a multiple of 16).
__device__ __forceinline__ void prefetch_l2_bulk(const void *p, uint32_t bytes) {
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(p), "r"(bytes) : "memory");
}
// ... for a word table (streamed: evict_first)
__device__ __forceinline__ void prefetch_l2_table(const void *p, uint32_t bytes) {
#if LDA_L2HINT
    asm volatile("cp.async.bulk.prefetch.L2.global.L2::cache_hint [%0], %1, %2;" ::"l"(p), "r"(bytes),
                 "l"(pol_evict_first())
                 : "memory");
#else
    prefetch_l2_bulk(p, bytes);
#endif
}

// Word-major position of virtual index v of a word whose item spans runs
// [lo, hi) (hi = the word's sentinel): binary search of the run holding v.
__device__ __forceinline__ uint32_t run_position(const Seg *__restrict__ segs, uint32_t lo, uint32_t hi,
                                                 uint32_t v) {
    while (hi - lo > 1) {
        const uint32_t mid = (lo + hi) >> 1;
        if (segs[mid].vstart <= v) lo = mid;
        else hi = mid;
    }
    return segs[lo].pos + (v - segs[lo].vstart);
}

// ---------------------------------------------------------------------------
// a1: random initial assignment (L377-379; X10): z = (x0·K) >> 32, t = 0.
// ---------------------------------------------------------------------------
__global__ void init_kernel(const SampleChunk *__restrict__ chunks, int64_t n_chunks,
                            const Seg *__restrict__ segs, const uint32_t *__restrict__ tok_crank,
                            uint16_t *__restrict__ z, uint32_t K, uint32_t k0, uint32_t k1) {
    for (int64_t ci = blockIdx.x; ci < n_chunks; ci += gridDim.x) {
        const SampleChunk ch = chunks[ci];
        for (uint32_t j = threadIdx.x; j < ch.count; j += blockDim.x) {
            const uint32_t p = run_position(segs, ch.seg0, ch.segN, ch.vbegin + j);
            const uint32_t x0 = philox_x0(ch.c_base + tok_crank[p], 0u, k0, k1);
            z[p] = static_cast<uint16_t>((static_cast<uint64_t>(x0) * K) >> 32);
        }
    }
}

// The same draw for the tile samplers' layout: token pos + j of an item has
// canonical rank crank0 + j.
__global__ void init_tile_kernel(const TileItem *__restrict__ items, int64_t n_items,
                                 const uint64_t *__restrict__ cbase, uint16_t *__restrict__ z, uint32_t K,
                                 uint32_t k0, uint32_t k1) {
    for (int64_t ci = blockIdx.x; ci < n_items; ci += gridDim.x) {
        const TileItem it = items[ci];
        const uint64_t c0 = cbase[it.word] + it.crank0;
        for (uint32_t j = threadIdx.x; j < it.n; j += blockDim.x) {
            const uint32_t x0 = philox_x0(c0 + j, 0u, k0, k1);
            z[it.pos + j] = static_cast<uint16_t>((static_cast<uint64_t>(x0) * K) >> 32);
        }
    }
}

// ---------------------------------------------------------------------------
// a2: sweep prologue, denom[k] = n_k + Vβ  (fp64, Eq. 1 / Eq. 8 denominator).
// ---------------------------------------------------------------------------
__global__ void prologue_kernel(const int32_t *__restrict__ nk, int K, double Vbeta,
                                double *__restrict__ denom) {
    for (int k = blockIdx.x * blockDim.x + threadIdx.x; k < K; k += gridDim.x * blockDim.x)
        denom[k] = static_cast<double>(nk[k]) + Vbeta;
}

// ---------------------------------------------------------------------------
// a3 + a4: the sampling kernel.
//
// Persistent CTAs pull word chunks from a queue (heavy-first, L1203-1221).
// Per chunk the CTA builds, in shared memory, p*(k) = (n_wk + β)/(n_k + Vβ)
// (Eq. 8, one division per topic, the oracle's exact expression) and the
// inclusive prefix P of α·p*(k) (the dense bucket p2 of Eq. 6, shared by all
// tokens of the word: Fig. 6).  Then every thread draws its own
// tokens (one sampler per lane):
//   pass 1   S = Σ_j c_j·p*(t_j) over the doc's θ row (p1 of Eq. 6, Eq. 7),
//            32-byte row blocks, zero-mass padding, no per-entry bounds check
//   draw     x = U·(S+Q), U = x0·2^-32 from Philox(seed; c, t) (X4, X8, X9)
//   sparse   x < S: rescan the row, first entry with prefix > x (X5, X6)
//   dense    else: binary search of the first k with S + P[k] > x (Fig. 5)
// θ rows: word 0 = nnz, words 1..nnz = topic << 18 | count (ascending topics,
// X7), zero words up to the next 32-byte boundary.
// ---------------------------------------------------------------------------
struct SweepArgs {
    const SampleChunk *chunks;
    int64_t n_chunks;
    const Seg *segs;
    const uint32_t *tok_row;
    const uint32_t *tok_crank;
    uint16_t *z;
    const uint4 *rows;
    const int32_t *nwk;
    const int32_t *nk;
    const double *denom;
    uint32_t *counter;
    int32_t *nwk_next;  // fused recount target rows (V*K), or null
    int32_t *nk_next;   // and its n_k
    double *gscratch;  // non-null when the K-length arrays do not fit in smem
    int K;
    double alpha, beta, Vbeta;
    uint32_t t;
    uint32_t key0[10], key1[10];  // Philox key schedule (seed + r·W)
};

__device__ __forceinline__ uint32_t philox_x0_sched(uint64_t c, uint32_t t, const uint32_t *k0,
                                                    const uint32_t *k1) {
    uint32_t c0 = static_cast<uint32_t>(c), c1 = static_cast<uint32_t>(c >> 32), c2 = t, c3 = 0u;
#pragma unroll
    for (int r = 0; r < 10; ++r) {
        const uint32_t hi0 = __umulhi(0xD2511F53u, c0), lo0 = 0xD2511F53u * c0;
        const uint32_t hi1 = __umulhi(0xCD9E8D57u, c2), lo1 = 0xCD9E8D57u * c2;
        c0 = hi1 ^ c1 ^ k0[r];
        c1 = lo1;
        c2 = hi0 ^ c3 ^ k1[r];
        c3 = lo0;
    }
    return c0;
}

template <bool EXCL, int TS>
struct Mass {
    // mass of one θ entry e = topic << TS | count under the word's p*
    __device__ __forceinline__ static double fma_into(uint32_t e, const double *__restrict__ pstar, int zo,
                                                      double po_new, double acc) {
        const uint32_t tp = e >> TS;
        uint32_t cn = e & 0xFFFFu;
        double p = pstar[tp];
        if (EXCL && static_cast<int>(tp) == zo && cn != 0u) {
            cn -= 1u;
            p = po_new;
        }
        return fma(static_cast<double>(cn), p, acc);
    }
};

// SMEMP: p*/P in shared memory (LDS addressing); else in a global scratch
// slice per CTA (large K).
template <bool EXCL, bool SMEMP, int TS = kTS>
__global__ void __launch_bounds__(kSweepThreads, LDA_SWEEP_MINB) sweep_kernel(SweepArgs a) {
    extern __shared__ double smem_d[];
    __shared__ int s_ci;
    __shared__ double s_wtot[kSweepThreads / 32];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int K = a.K;
    // smem: [blkC: kMaxBlk x 256 fp64][p*: K][P: K][hist: K i32][nk partial: K i32]
    // (SMEMP = false: p*/P in a global scratch slice, no fused recount)
    double *blkC = smem_d;
    double *pstar = SMEMP ? smem_d + kMaxBlk * kSweepThreads : a.gscratch + static_cast<size_t>(blockIdx.x) * 2 * K;
    double *P = pstar + K;
    int *hist = reinterpret_cast<int *>(smem_d + kMaxBlk * kSweepThreads + 2 * K);
    int *nkp = hist + K;
    if (SMEMP) {
        for (int k = tid; k < 2 * K; k += kSweepThreads) hist[k] = 0;
    }
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
                    const double ps = (static_cast<double>(__ldg(nwk_row + k)) + a.beta) / __ldg(a.denom + k);
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

        // One sampler per lane; each thread draws tokens j, j+256, ...  The
        // row is streamed in 32-byte blocks (one 256-bit load per block per
        // lane, sm_100 LDG.256) through a ring of kRing blocks held in
        // registers; words past nnz in the last block are zero.
        uint32_t pn = 0, rown = 0;
        if (static_cast<uint32_t>(tid) < ch.count) {
            pn = run_position(a.segs, ch.seg0, ch.segN, ch.vbegin + tid);
            rown = __ldg(a.tok_row + pn);
        }
        for (uint32_t j = tid; j < ch.count; j += kSweepThreads) {
            const uint32_t p = pn;
            const uint32_t *rw = reinterpret_cast<const uint32_t *>(a.rows) + static_cast<size_t>(rown) * 8;
            Blk8 q[kRing];
            q[0] = ld_nc_v8(rw);           // block 0: nnz + 7 entries
            const uint32_t jn = j + kSweepThreads;
            if (jn < ch.count) {
                pn = run_position(a.segs, ch.seg0, ch.segN, ch.vbegin + jn);
                rown = __ldg(a.tok_row + pn);
            }
            const uint32_t x0 = philox_x0_sched(ch.c_base + __ldg(a.tok_crank + p), a.t, a.key0, a.key1);
            int zo = 0;
            double po_new = 0.0, delta = 0.0;
            if (EXCL) {
                zo = static_cast<int>(a.z[p]);
                po_new = (static_cast<double>(nwk_row[zo] - 1) + a.beta) /
                         (static_cast<double>(a.nk[zo] - 1) + a.Vbeta);
                delta = a.alpha * po_new - a.alpha * pstar[zo];
            }
            const uint32_t len = q[0].w[0];
            const uint32_t nblk = (len + 8u) >> 3;   // 32-byte blocks holding words 0..len
#pragma unroll
            for (int i = 1; i < kRing; ++i)
                if (static_cast<uint32_t>(i) < nblk) q[i] = ld_nc_v8(rw + 8 * i);
            int z;
            // pass 1: S over the row, block-end prefixes to smem
            double S = 0.0;
#pragma unroll
            for (int e = 1; e < 8; ++e) S = Mass<EXCL, TS>::fma_into(q[0].w[e], pstar, zo, po_new, S);
            blkC[tid] = S;
            if (static_cast<uint32_t>(kRing) < nblk) q[0] = ld_nc_v8(rw + 8 * kRing);
            // blocks 1 .. nblk-1, ring slot (b % kRing)
            for (uint32_t base = 0; base < nblk; base += kRing) {
#pragma unroll
                for (int i = 0; i < kRing; ++i) {
                    const uint32_t b = base + i;
                    if (b == 0) continue;
                    if (b >= nblk) break;
                    const Blk8 u = q[i];
                    const uint32_t nx = b + kRing;
                    if (nx < nblk) q[i] = ld_nc_v8(rw + 8 * nx);
#pragma unroll
                    for (int e = 0; e < 8; ++e) S = Mass<EXCL, TS>::fma_into(u.w[e], pstar, zo, po_new, S);
                    if (b < kMaxBlk) blkC[b * kSweepThreads + tid] = S;
                }
            }
            const double U = static_cast<double>(x0) * 2.3283064365386962890625e-10;  // x0 · 2^-32
            const double x = U * (S + (EXCL ? Q + delta : Q));
            if (x < S) {
                // sparse bucket (p1): the first block whose end prefix exceeds x,
                // then the identical recomputation inside it: first C > x
                const uint32_t nb = nblk < kMaxBlk ? nblk : kMaxBlk;
                uint32_t b = 0;
                while (b < nb && !(blkC[b * kSweepThreads + tid] > x)) ++b;
                double C = b == 0 ? 0.0 : blkC[(b - 1) * kSweepThreads + tid];
                z = -1;
#define LDA_STEP(e)                                                   \
    {                                                                 \
        C = Mass<EXCL, TS>::fma_into((e), pstar, zo, po_new, C);      \
        if (z < 0 && C > x) z = static_cast<int>((e) >> TS);           \
    }
                for (; z < 0 && b < nblk; ++b) {  // one block, or a linear tail past kMaxBlk
                    const Blk8 u = ld_nc_v8(rw + 8 * b);
                    if (b > 0) LDA_STEP(u.w[0])
#pragma unroll
                    for (int e = 1; e < 8; ++e) LDA_STEP(u.w[e])
                }
#undef LDA_STEP
                if (z < 0) z = K - 1;  // unreachable: the last entry's prefix is S > x
            } else {
                // dense bucket (p2): first k with S + P[k] (+Δ for k >= zo) > x
                int lo = 0, hi = K - 1;
                while (lo < hi) {
                    const int mid = (lo + hi) >> 1;
                    double pk = P[mid];
                    if (EXCL && mid >= zo) pk += delta;
                    if (S + pk > x) hi = mid;
                    else lo = mid + 1;
                }
                z = lo;  // K-1 also when x >= S + Q by rounding (X6 fallback)
            }
            a.z[p] = static_cast<uint16_t>(z);
            if (SMEMP) atomicAdd(&hist[z], 1);
        }
        __syncthreads();
        if (SMEMP) {
            // fused n_wk recount (ϕ update, L1273-1285): this chunk's topic
            // histogram -> the word's row of the next n_wk; atomics only when
            // the word is split over several chunks
            int32_t *row = a.nwk_next + static_cast<size_t>(ch.word) * K;
            const bool split = (ch.pad & 1u) != 0u;
            for (int k = tid; k < K; k += kSweepThreads) {
                const int h = hist[k];
                if (split) {
                    if (h) atomicAdd(row + k, h);
                } else {
                    row[k] = h;
                }
                nkp[k] += h;
                hist[k] = 0;
            }
        }
        __syncthreads();
    }
    if (SMEMP) {
        for (int k = tid; k < K; k += kSweepThreads)
            if (nkp[k]) atomicAdd(a.nk_next + k, nkp[k]);
    }
}

// count (low 16 bits of a θ entry) as float, exactly: bits 0x4B00:count = 2^23 + c
__device__ __forceinline__ float count_f32(uint32_t e) {
    return __uint_as_float(__byte_perm(e, 0x4B00u, 0x5410)) - 8388608.0f;
}
// (PRMT + FADD; measured faster on B200 than LOP3 + I2FP.F32.U32: -0.5 %)
// the line sum of line L from its four block sums (the quad's order)
__device__ __forceinline__ float line_sum(const float *blk, uint32_t L) {
    const float4 b = *reinterpret_cast<const float4 *>(blk + 4 * L);
    return (b.x + b.y) + (b.z + b.w);
}
// the entry's topic in an fp32 table: byte offset e >> 16 = 4·topic
__device__ __forceinline__ float tab32(const float *__restrict__ p32, uint32_t e) {
    return *reinterpret_cast<const float *>(reinterpret_cast<const char *>(p32) + (e >> 16));
}
__device__ __forceinline__ float entry_mass32(uint32_t e, const float *__restrict__ p32, float acc) {
    return fmaf(count_f32(e), tab32(p32, e), acc);
}

// Packed fp32 pairs (Blackwell FFMA2 / FADD2 / FMUL2: two IEEE fp32
// operations per instruction, each rounded as its scalar form -- the two
// FFMA chains of a block sum below stay bit-identical).
typedef unsigned long long f32x2;
__device__ __forceinline__ f32x2 f2_pack(float a, float b) {
    f32x2 r;
    asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(a), "f"(b));
    return r;
}
__device__ __forceinline__ f32x2 f2_add(f32x2 a, f32x2 b) {
    f32x2 r;
    asm("add.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
    return r;
}
__device__ __forceinline__ f32x2 f2_mul(f32x2 a, f32x2 b) {
    f32x2 r;
    asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
    return r;
}
__device__ __forceinline__ f32x2 f2_fma(f32x2 a, f32x2 b, f32x2 c) {
    f32x2 r;
    asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r) : "l"(a), "l"(b), "l"(c));
    return r;
}
__device__ __forceinline__ float f2_hsum(f32x2 a) {
    float x, y;
    asm("mov.b64 {%0, %1}, %2;" : "=f"(x), "=f"(y) : "l"(a));
    return x + y;
}
// the counts of entries e0, e1 as an fp32 pair: (2^23 + c) - 2^23, exact
__device__ __forceinline__ f32x2 count_f32x2(uint32_t e0, uint32_t e1) {
    return f2_add(f2_pack(__uint_as_float(__byte_perm(e0, 0x4B00u, 0x5410)),
                          __uint_as_float(__byte_perm(e1, 0x4B00u, 0x5410))),
                  f2_pack(-8388608.0f, -8388608.0f));
}
// the masses c·p32(t) of entries e0, e1, added to the pair acc
__device__ __forceinline__ f32x2 mass_f32x2(uint32_t e0, uint32_t e1, const float *__restrict__ p32, f32x2 acc) {
    return f2_fma(count_f32x2(e0, e1), f2_pack(tab32(p32, e0), tab32(p32, e1)), acc);
}

// ---------------------------------------------------------------------------
// a3 + a4, tile sampler (sampler 2, the default).
//
// Work items are (word, doc tile) runs: the tokens of word w inside one tile
// of documents, contiguous in the word-major stream (L1189-1191), at most
// chunk_tokens each, queued tile by tile (heavy-first inside a tile,
// L1203-1221).  All warps of the GPU work on the same tile at a time, so the
// θ rows the tile's tokens gather (tens of MB) are read from HBM about once
// and re-read from the 126 MB L2.  Each WARP owns an item (no CTA barriers):
//   prologue  p32(k) = (n_wk + β)·fl32(1/(n_k + Vβ)) and the inclusive
//             prefix P32 of α·p32 in the warp's shared memory (Eq. 8 and the
//             dense bucket p2 of Eq. 6, shared by the word's tokens, Fig. 6)
//   walk      32 tokens per batch; a quad (4 lanes) walks one token's θ row
//             one 128-byte line per step (lane `sub` holds entries
//             8·sub .. 8·sub+7: one 256-bit load, one L1 wavefront per line),
//             S = Σ c_j·p32(t_j) (p1 of Eq. 6-7) with the prefix at every
//             8-entry block end kept in smem (first kTBlk blocks)
//   draw      lane per token: x = U·(S+Q), U = x0·2^-32 from Philox (X4, X8,
//             X9); sparse: binary search of the block-end prefixes, rescan of
//             one block (first C > x, X5/X6); dense: binary search of P32
//   verify    every comparison above is taken only if its margin exceeds a
//             rigorous bound on the fp32 error (γ·u terms below); a token
//             with any closer comparison is redrawn by the warp in fp64 from
//             the counts (draw_exact_warp) -- so the draw is the exact-
//             arithmetic draw of Eq. 1, i.e. the oracle's up to fp64 rounding
//             at a CDF boundary (excused within 1e-6)
//   recount   z stored, n_wk of the next sweep += 1 (one global reduction per
//             distinct topic of the batch), n_k in a per-CTA smem histogram
//             (the ϕ update, L1273-1285, fused)
// ---------------------------------------------------------------------------
#ifndef LDA_TRING
#define LDA_TRING 3
#endif
#ifndef LDA_CTA_NBUF_MAX
#define LDA_CTA_NBUF_MAX 3   // large-K CTA sampler: table buffers per CTA (at most; 3: 16 warps, +2.5 % over 4 at K = 8192)
#endif
#ifndef LDA_CTA_MIN_WARPS
#define LDA_CTA_MIN_WARPS 12  // ...as long as at least this many warps fit beside them
#endif
#ifndef LDA_TRING_GNK
#define LDA_TRING_GNK 3  // the large-K CTA sampler's ring (4: +0.5 % at K = 8192 alone, -0.2 % with the early line-table reads)
#endif
#ifndef LDA_F32X2
#define LDA_F32X2 1  // the walk's block sums with packed fp32 pairs (FFMA2)
#endif
#ifndef LDA_LCACHE
#define LDA_LCACHE 1  // the draw keeps the prefixes after the first 3 θ-row lines from the S pass
#endif
#ifndef LDA_BALLOT_SCAN
#define LDA_BALLOT_SCAN 1  // the batch head's line-count prefix by ballots (K < 2016)
#endif
#ifndef LDA_NC8
#define LDA_NC8 1  // the dense chunk search specialised for 8 chunks (K = 1024)
#endif
#ifndef LDA_LSEL
#define LDA_LSEL 1  // the draw's line selection (first three lines) branch-free
#endif
#ifndef LDA_BSEL
#define LDA_BSEL 1  // the draw's block search branch-free
#endif
#ifndef LDA_DENSE4
#define LDA_DENSE4 1  // the dense in-chunk search 4-ary (4 dependent loads instead of 7)
#endif
#ifndef LDA_TILE_WPC
#define LDA_TILE_WPC 8
#endif
#ifndef LDA_TILE_LMAX
#define LDA_TILE_LMAX 160
#endif
#ifndef LDA_TILE_MINB
#define LDA_TILE_MINB 2
#endif
#ifndef LDA_TILE_MAXK
#define LDA_TILE_MAXK 4096
#endif
constexpr int kTileMaxK = LDA_TILE_MAXK;

#ifndef LDA_TILE_STATS
#define LDA_TILE_STATS 0
#endif

#if LDA_TILE_STATS
// diagnostics build only: batches, tokens, θ-row lines walked, distinct rows, walk steps
__device__ unsigned long long g_tile_stats[8];
extern "C" int lda_debug_tile_stats(unsigned long long *out, int reset) {
    cudaError_t e = cudaMemcpyFromSymbol(out, g_tile_stats, sizeof(g_tile_stats));
    if (e == cudaSuccess && reset) {
        unsigned long long z[8] = {0, 0, 0, 0, 0, 0, 0, 0};
        e = cudaMemcpyToSymbol(g_tile_stats, z, sizeof(z));
    }
    return e;
}
#endif
struct TileArgs {
    const TileItem *items;
    int64_t n_items;
    const uint64_t *cbase;     // V: canonical index of the rank's first token of each word
    const uint32_t *tok_row;   // word-major: θ row of the token's doc (32-byte units, 128-byte aligned)
    uint16_t *z;
    const uint32_t *rows;
    const int32_t *nwk;        // frozen counts (V*K, n_k after)
    const double *denom;       // K: n_k + Vβ
    uint32_t *counter;
    int32_t *nwk_next;         // zeroed next counts, V*K
    int32_t *nk_next;          // and n_k
    unsigned long long *n_exact;
    int K;
    double alpha, beta;
    int lmax;                  // max θ-row lines per batch (per-warp smem)
    double slack;              // multiplier of every certification bound (1; > 1 only in tests)
    const char *wtab;          // word tables (word_table_kernel), wt_bytes per word
    uint32_t wt_bytes;
    int nbuf;                  // sweep_tile_cta_kernel: table buffers per CTA
    int recount;               // 1: the ϕ update fused here; 0: recount_kernel after the sweep
    // f2 sparse word rows (sweep_tile_cta_kernel, compact tables): see SparseRows
    const uint32_t *sp_off;    // V+1, null = off
    const uint32_t *sp_nnz;
    const uint32_t *sp_ent;
    const float *s32;
    uint32_t t;
    uint32_t key0[10], key1[10];
};

__device__ __forceinline__ double warp_sum_d(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(kFull, v, o);
    return v;
}
__device__ __forceinline__ double warp_incl_scan_d(double v, int lane) {
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const double y = __shfl_up_sync(kFull, v, o);
        if (lane >= o) v += y;
    }
    return v;
}
__device__ __forceinline__ double pstar64(const int32_t *nwk_row, const double *denom, double beta, uint32_t k) {
    return (static_cast<double>(__ldg(nwk_row + k)) + beta) / __ldg(denom + k);
}

// Exact (fp64) draw of one token by the whole warp, from the counts in global
// memory: p*(k) = (n_wk+β)/(n_k+Vβ) as the oracle computes it, S over the
// doc row, x = U·(S+Q), then the first bin of [sparse ‖ dense] whose prefix
// exceeds x (X4-X6).  Q and the dense prefix at every group start come from
// the word's table (B[g] = fp64 prefix of α·p* before group g of gsz topics,
// B[G] = Q, built by word_table_kernel): the dense search jumps to the group
// holding x and scans it with the exact p*, O(log G + gsz) instead of O(K).
// Only the summation order (and p* by reciprocal inside B) differs from the
// oracle's: fp64 rounding, far below the north_star's 1e-6 excuse.
__device__ __noinline__ int draw_exact_warp(const int32_t *nwk_row, const double *denom, const uint32_t *rw,
                                            uint32_t nnz, uint32_t x0, int K, double alpha, double beta,
                                            const double *B, int G, int gsz) {
    const int lane = threadIdx.x & 31;
    const double Q = B[G];
    double s = 0.0;
    for (uint32_t j = 1 + lane; j <= nnz; j += 32) {
        const uint32_t e = __ldg(rw + j);
        s = fma(static_cast<double>(e & 0xFFFFu), pstar64(nwk_row, denom, beta, e >> kTS), s);
    }
    const double S = warp_sum_d(s);
    const double x = static_cast<double>(x0) * 2.3283064365386962890625e-10 * (S + Q);
    if (x < S) {
        double carry = 0.0;
        for (uint32_t j0 = 1; j0 <= nnz; j0 += 32) {
            const uint32_t j = j0 + lane;
            double m = 0.0;
            uint32_t tp = 0;
            if (j <= nnz) {
                const uint32_t e = __ldg(rw + j);
                tp = e >> kTS;
                m = static_cast<double>(e & 0xFFFFu) * pstar64(nwk_row, denom, beta, tp);
            }
            const double c = carry + warp_incl_scan_d(m, lane);
            const unsigned hit = __ballot_sync(kFull, j <= nnz && m > 0.0 && c > x);
            if (hit) return static_cast<int>(__shfl_sync(kFull, tp, __ffs(hit) - 1));
            carry = __shfl_sync(kFull, c, 31);
        }
        return K - 1;
    }
    // the last group g with S + B[g] <= x (uniform over the warp)
    int g = 0;
    for (int n = G; n > 1;) {
        const int h = n >> 1;
        if (S + B[g + h] <= x) g += h;
        n -= h;
    }
    double carry = S + B[g];
    for (int k0 = g * gsz; k0 < K; k0 += 32) {
        const int k = k0 + lane;
        const double m = k < K ? alpha * pstar64(nwk_row, denom, beta, k) : 0.0;
        const double c = carry + warp_incl_scan_d(m, lane);
        const unsigned hit = __ballot_sync(kFull, k < K && c > x);
        if (hit) return k0 + __ffs(hit) - 1;
        carry = __shfl_sync(kFull, c, 31);
    }
    return K - 1;
}

// Positive normal fp32 <-> fp64 by bit manipulation (ALU pipe instead of the
// conversion unit).  f2d_pos is exact; d2f_trunc truncates (relative error
// < 2^-23); values below 2^-126 map to 0.
__device__ __forceinline__ double f2d_pos(float f) {
    const uint32_t b = __float_as_uint(f);
    const uint32_t hi = b ? (b >> 3) + 0x38000000u : 0u;
    return __hiloint2double(static_cast<int>(hi), static_cast<int>(b << 29));
}
__device__ __forceinline__ float d2f_trunc(double d) {
    const uint32_t hi = static_cast<uint32_t>(__double2hiint(d)), lo = static_cast<uint32_t>(__double2loint(d));
    return hi < 0x38100000u ? 0.0f : __uint_as_float(((hi - 0x38000000u) << 3) | (lo >> 29));
}
// n (0 <= n < 2^31) as double, exactly: (2^52 + n) - 2^52
__device__ __forceinline__ double i2d_pos(int n) {
    return __hiloint2double(0x43300000, n) - 4503599627370496.0;
}

// a3, hoisted out of the sampler: the word table of every word, built once
// per sweep from the frozen counts (Eq. 8).  p*(k) = (n_wk + β)·(1/(n_k + Vβ))
// in fp64; p32 = its truncation to fp32 (relative error < 2u, u = 2^-24) for
// the sparse walk; the dense prefix of α·p* in two levels: Pc[c] = Σ over
// the 128-topic chunks before c (fp64), L32[k] = the prefix inside k's chunk
// (fp64, truncated to fp32: error < 2u·L32), Pc[NC] = Q = Σ_k α·p*(k).
// Layout per word (wt_bytes, a multiple of 16): [Pc: NC+1 doubles, padded
// to an even count][p32: K4 floats][L32: K4 floats].  One warp per word;
// lane l holds k = 128c + 4l .. 4l+3 of chunk c.
// L32 holds whole 128-topic chunks, groups of 4 entries swizzled by the chunk
// index (k ^ ((c & 7) << 2)): the dense binary searches of lanes in different
// chunks probe the same in-chunk offsets, which would otherwise all fall in
// one shared-memory bank.
__host__ __device__ constexpr int tab_nc2(int K) { return ((K + 127) / 128 + 2) / 2 * 2; }
__host__ __device__ constexpr size_t tab_bytes(int K) {
    return static_cast<size_t>(tab_nc2(K)) * 8 + static_cast<size_t>(4) * ((K + 3) & ~3) +
           static_cast<size_t>(4) * 128 * ((K + 127) / 128);
}
__host__ __device__ constexpr int l32_idx(int k) { return k ^ (((k >> 7) & 7) << 2); }
// Compact layout (the large-K CTA sampler, which keeps several tables per
// CTA): [Pg: fp64 prefix of α·p* at the start of every 32-topic group, then
// Pg[G] = Q, padded to an even count][p32: K4 floats] -- the in-group prefix
// is summed on the fly from p32 (at most 32 terms).
__host__ __device__ constexpr int tab_g2(int K) { return ((K + 31) / 32 + 2) / 2 * 2; }
__host__ __device__ constexpr size_t tab_bytes_compact(int K) {
    return static_cast<size_t>(tab_g2(K)) * 8 + static_cast<size_t>(4) * ((K + 3) & ~3);
}

// f2 (SparseLDA's split of p* = β·inv(k) + n_wk·inv(k), ref [32], L999):
// sparse word rows.  A word with sp_off[w+1] > sp_off[w] ("rare": few tokens
// against K) gets no p32 row in its table -- only Pg -- but the list of its
// nonzero topics (topic, p32(topic)) in sp_ent[2·sp_off[w] ..], ascending,
// count in sp_nnz[w]; the sampler rebuilds its p32 row in shared memory from
// the smoothing row s32[k] = fl32(β·inv(k)) (shared by all words, written
// here by block 0) plus those entries -- bit-identical to the dense row.
struct SparseRows {
    const uint32_t *off;  // V+1 (null: off)
    uint32_t *nnz;        // V
    uint32_t *ent;        // 2 words per entry: topic, p32 bits
    float *s32;           // K4: fl32(β·inv(k)), zero padding
};

template <bool VEC, bool COMPACT>
__global__ void word_table_kernel(const int32_t *__restrict__ nwk, const double *__restrict__ denom, int V, int K,
                                  double alpha, double beta, char *__restrict__ tab, SparseRows sp) {
    extern __shared__ double inv64[];
    const int lane = threadIdx.x & 31;
    for (int k = threadIdx.x; k < K; k += blockDim.x) inv64[k] = 1.0 / denom[k];
    __syncthreads();
    const int K4 = (K + 3) & ~3;
    if (COMPACT && sp.off && blockIdx.x == 0)
        for (int k = threadIdx.x; k < K4; k += blockDim.x) sp.s32[k] = k < K ? d2f_trunc((0.0 + beta) * inv64[k]) : 0.0f;
    const size_t wt = COMPACT ? tab_bytes_compact(K) : tab_bytes(K);
    const int nwarp = gridDim.x * (blockDim.x >> 5);
    for (int w = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); w < V; w += nwarp) {
        const int32_t *nwk_row = nwk + static_cast<size_t>(w) * K;
        double *Pc = reinterpret_cast<double *>(tab + wt * w);
        float *p32 = reinterpret_cast<float *>(Pc + (COMPACT ? tab_g2(K) : tab_nc2(K)));
        float *L32 = p32 + K4;
        // f2: a sparse word's nonzero topics go to its list instead of a p32 row
        uint32_t *ent = nullptr;
        uint32_t nz = 0;
        if (COMPACT && sp.off) {
            const uint32_t o0 = __ldg(sp.off + w), o1 = __ldg(sp.off + w + 1);
            if (o1 > o0) ent = sp.ent + 2 * static_cast<size_t>(o0);
        }
        double carry = 0.0;
        // one 128-topic chunk (lane l: topics k0 + 4l .. 4l+3; VEC: their counts n)
        auto chunk = [&](const int k0, const int c, const int4 n) {
            const int k = k0 + 4 * lane;
            double a4[4] = {0.0, 0.0, 0.0, 0.0};
            if (VEC) {
                if (k < K || (COMPACT && ent)) {
                    float f4[4] = {0.0f, 0.0f, 0.0f, 0.0f};
                    if (k < K) {
                        const double p0 = (i2d_pos(n.x) + beta) * inv64[k], p1 = (i2d_pos(n.y) + beta) * inv64[k + 1];
                        const double p2 = (i2d_pos(n.z) + beta) * inv64[k + 2],
                                     p3 = (i2d_pos(n.w) + beta) * inv64[k + 3];
                        f4[0] = d2f_trunc(p0);
                        f4[1] = d2f_trunc(p1);
                        f4[2] = d2f_trunc(p2);
                        f4[3] = d2f_trunc(p3);
                        if (!(COMPACT && ent)) *reinterpret_cast<float4 *>(p32 + k) = make_float4(f4[0], f4[1], f4[2], f4[3]);
                        a4[0] = alpha * p0;
                        a4[1] = alpha * p1;
                        a4[2] = alpha * p2;
                        a4[3] = alpha * p3;
                    }
                    if (COMPACT && ent) {
                        // the nonzero topics of this 128-topic chunk, in topic order
                        const int cnt = (n.x != 0) + (n.y != 0) + (n.z != 0) + (n.w != 0);
                        int incl = cnt;
#pragma unroll
                        for (int o = 1; o < 32; o <<= 1) {
                            const int y = __shfl_up_sync(kFull, incl, o);
                            if (lane >= o) incl += y;
                        }
                        uint32_t j = nz + static_cast<uint32_t>(incl - cnt);
                        const int nn[4] = {n.x, n.y, n.z, n.w};
#pragma unroll
                        for (int e = 0; e < 4; ++e)
                            if (nn[e] != 0) {
                                ent[2 * j] = static_cast<uint32_t>(k + e);
                                ent[2 * j + 1] = __float_as_uint(f4[e]);
                                ++j;
                            }
                        nz += static_cast<uint32_t>(__shfl_sync(kFull, incl, 31));
                    }
                }
            } else {
#pragma unroll
                for (int e = 0; e < 4; ++e)
                    if (k + e < K) {
                        const double pe = (i2d_pos(__ldg(nwk_row + k + e)) + beta) * inv64[k + e];
                        p32[k + e] = d2f_trunc(pe);
                        a4[e] = alpha * pe;
                    }
            }
            const double l0 = a4[0], l1 = l0 + a4[1], l2 = l1 + a4[2], l3 = l2 + a4[3];
            double incl = l3;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const double y = __shfl_up_sync(kFull, incl, o);
                if (lane >= o) incl += y;
            }
            double excl = __shfl_up_sync(kFull, incl, 1);
            if (lane == 0) excl = 0.0;
            if (COMPACT) {
                // lane 8g starts group g of this chunk: its base is the group's prefix
                if ((lane & 7) == 0 && k < K) Pc[4 * c + (lane >> 3)] = carry + excl;
            } else {
                const float f0 = d2f_trunc(excl + l0), f1 = d2f_trunc(excl + l1);
                const float f2 = d2f_trunc(excl + l2), f3 = d2f_trunc(excl + l3);
                if (VEC) {
                    if (k < K) *reinterpret_cast<float4 *>(L32 + l32_idx(k)) = make_float4(f0, f1, f2, f3);
                } else {
                    const float ff[4] = {f0, f1, f2, f3};
#pragma unroll
                    for (int e = 0; e < 4; ++e)
                        if (k + e < K) L32[l32_idx(k + e)] = ff[e];
                }
                if (lane == 0) Pc[c] = carry;
            }
            carry += __shfl_sync(kFull, incl, 31);
        };
        if (VEC) {
            // the counts of 4 chunks in flight at a time (the chunks' fp64
            // scans are a serial chain: without this the loads wait in it)
            for (int k00 = 0; k00 < K; k00 += 512) {
                int4 nn[4];
#pragma unroll
                for (int u = 0; u < 4; ++u) {
                    const int k = k00 + 128 * u + 4 * lane;
                    nn[u] = k < K ? __ldg(reinterpret_cast<const int4 *>(nwk_row + k)) : make_int4(0, 0, 0, 0);
                }
#pragma unroll
                for (int u = 0; u < 4; ++u)
                    if (k00 + 128 * u < K) chunk(k00 + 128 * u, k00 / 128 + u, nn[u]);
            }
        } else {
            for (int k0 = 0, c = 0; k0 < K; k0 += 128, ++c) chunk(k0, c, make_int4(0, 0, 0, 0));
        }
        // zero the padding so that the table bytes are deterministic
        if (COMPACT) {
            const int G = (K + 31) / 32;
            if (lane == 0) Pc[G] = carry;
            if (lane == 1 && tab_g2(K) > G + 1) Pc[tab_g2(K) - 1] = 0.0;
        } else {
            if (lane == 0) Pc[(K + 127) / 128] = carry;
            if (lane == 1 && tab_nc2(K) > (K + 127) / 128 + 1) Pc[tab_nc2(K) - 1] = 0.0;
            for (int k = K + lane; k < 128 * ((K + 127) / 128); k += 32) L32[l32_idx(k)] = 0.0f;
        }
        if (COMPACT && ent) {
            if (lane == 0) sp.nnz[w] = nz;
        } else {
            for (int k = K + lane; k < K4; k += 32) p32[k] = 0.0f;
        }
    }
}

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
    uint32_t done = 0;
    while (!done) {
        asm volatile(
            "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
            : "=r"(done)
            : "r"(smem_u32(bar)), "r"(parity)
            : "memory");
    }
}
// Bulk copy (TMA engine, no LSU wavefronts) global -> this CTA's smem,
// completion counted on the mbarrier.
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *bar) {
#if LDA_L2HINT
    // word tables are streamed (read once per tile): evict_first in L2
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], "
        "%4;" ::"r"(smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol_evict_first())
        : "memory");
#else
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
            smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar))
        : "memory");
#endif
}

// Per-warp shared memory of the tile sampler (bytes): the word table, block
// sums, line table, per-token row / line base, mbarrier.
__host__ __device__ constexpr size_t tile_warp_bytes(int K, int lmax) {
    return tab_bytes(K) + static_cast<size_t>(lmax) * (16 + 4 + 4) + 32 * 4 + 16;
}

// Batch head of the tile sampler: up to 32 tokens whose θ rows have at most
// LM lines in total; consecutive tokens of one document -- a (word, doc)
// pair -- share the walk of its row.  Writes the line table (bits 0-30: θ
// row offset of the line in 32-byte units, bit 31: first line of its row) and
// puts the first R lines of the walk in flight.
struct TileHead {
    bool take, dup;
    int nb;
    uint32_t lsum, c0, nl;
};
template <int R>
__device__ __forceinline__ TileHead tile_head(const TileArgs &a, uint32_t row, uint32_t nnz, bool valid, int LM,
                                              uint32_t *lrow, Blk8 (&ring)[R], bool (&hdr)[R]) {
    const int lane = threadIdx.x & 31, q = lane >> 2, sub = lane & 3;
    TileHead h;
    const uint32_t prow = __shfl_up_sync(kFull, row, 1);
    h.dup = valid && lane > 0 && prow == row;
    h.nl = valid ? (nnz + 32u) >> 5 : 0u;  // 128-byte lines holding words 0..nnz
    const uint32_t nlw = h.dup ? 0u : h.nl;
    uint32_t incl = nlw;
#if LDA_BALLOT_SCAN
    if (a.K <= 2015) {
        // nlw < 64: the inclusive prefix by bit planes (six independent
        // ballots instead of five dependent shuffle rounds)
        const unsigned le = 0xFFFFFFFFu >> (31 - lane);
        incl = 0u;
#pragma unroll
        for (int bp = 0; bp < 6; ++bp) incl += static_cast<uint32_t>(__popc(__ballot_sync(kFull, (nlw >> bp) & 1u) & le)) << bp;
    } else
#endif
    {
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(kFull, incl, o);
            if (lane >= o) incl += y;
        }
    }
    h.take = valid && (incl <= static_cast<uint32_t>(LM) || lane == 0);
    h.nb = __popc(__ballot_sync(kFull, h.take));
    const uint32_t ls = __shfl_sync(kFull, incl, h.nb > 0 ? h.nb - 1 : 0);
    h.lsum = h.nb > 0 ? ls : 0u;
    const uint32_t c0 = incl - nlw;
    // a duplicate's lines are those of the last non-duplicate lane before it
    const unsigned heads = __ballot_sync(kFull, !h.dup);
    const int hl = 31 - __clz(heads & (0xFFFFFFFFu >> (31 - lane)));
    h.c0 = __shfl_sync(kFull, c0, hl);
    if (h.take && !h.dup) {
        for (uint32_t i = 0; i < h.nl; ++i) lrow[h.c0 + i] = (row + 4u * i) | (i == 0 ? 0x80000000u : 0u);
    }
    __syncwarp();
#pragma unroll
    for (int s2 = 0; s2 < R; ++s2) {
        const uint32_t L = q + 8u * s2;
#pragma unroll
        for (int e = 0; e < 8; ++e) ring[s2].w[e] = 0u;
        hdr[s2] = false;
        if (L < h.lsum) {
            const uint32_t lr = lrow[L];
            ring[s2] = ld_row_v8(a.rows + (static_cast<size_t>(lr & 0x7FFFFFFFu) + sub) * 8);
            hdr[s2] = sub == 0 && (lr >> 31);
        }
    }
    return h;
}

// The walk (p1 of Eq. 6): quad q takes lines q, q+8, ... of the batch; lane
// `sub` sums entries 8·sub .. 8·sub+7 of the line (two FFMA chains); the
// quad's line sum by two xor-shuffles.  Branch-free over the R lines in
// flight (a lane past the end sums stale entries and discards them).
// at_step2() runs once, at the start of the last step (the caller's prefetch hook).
// LR_EARLY: the refills' line-table entries are read before the block sums
// (their shared-load latency overlaps them; measured +0.4 % for the large-K
// CTA sampler, -0.3 % for the per-warp tile sampler)
template <int R, bool LR_EARLY = false, class F>
__device__ __forceinline__ void tile_walk(const TileArgs &a, uint32_t lsum, const uint32_t *lrow, Blk8 (&ring)[R],
                                          bool (&hdr)[R], const float *p32, float *blk, F &&at_step2) {
    const int lane = threadIdx.x & 31, q = lane >> 2, sub = lane & 3;
    bool hooked = false;
    for (uint32_t base = 0; base < lsum; base += 8u * R) {
        // the caller's prefetch hook at the start of the last step (or after
        // a single step): the loads it issues (the next batch's θ row
        // headers) depend on loads issued before the walk, which then have
        // all earlier steps to land (measured +1 % over the second step)
        if (base > 0 && base + 8u * R >= lsum) {
            at_step2();
            hooked = true;
        }
        float bs[R];
        uint32_t lrn[R];
        if (LR_EARLY) {
#pragma unroll
            for (int s2 = 0; s2 < R; ++s2) {
                const uint32_t Ln = base + 8u * (s2 + R) + q;
                lrn[s2] = Ln < lsum ? lrow[Ln] : 0u;
            }
        }
#pragma unroll
        for (int s2 = 0; s2 < R; ++s2) {
            const uint32_t w0 = hdr[s2] ? 0u : ring[s2].w[0];  // header word
#if LDA_F32X2
            // the two chains (even / odd entries) as one packed pair
            f32x2 sp = f2_mul(count_f32x2(w0, ring[s2].w[1]),
                              f2_pack(tab32(p32, w0), tab32(p32, ring[s2].w[1])));
            sp = mass_f32x2(ring[s2].w[2], ring[s2].w[3], p32, sp);
            sp = mass_f32x2(ring[s2].w[4], ring[s2].w[5], p32, sp);
            sp = mass_f32x2(ring[s2].w[6], ring[s2].w[7], p32, sp);
            bs[s2] = f2_hsum(sp);
#else
            float s0 = count_f32(w0) * tab32(p32, w0);
            float s1 = count_f32(ring[s2].w[1]) * tab32(p32, ring[s2].w[1]);
            s0 = entry_mass32(ring[s2].w[2], p32, s0);
            s1 = entry_mass32(ring[s2].w[3], p32, s1);
            s0 = entry_mass32(ring[s2].w[4], p32, s0);
            s1 = entry_mass32(ring[s2].w[5], p32, s1);
            s0 = entry_mass32(ring[s2].w[6], p32, s0);
            s1 = entry_mass32(ring[s2].w[7], p32, s1);
            bs[s2] = s0 + s1;
#endif
        }
#pragma unroll
        for (int s2 = 0; s2 < R; ++s2) {
            const uint32_t Ln = base + 8u * (s2 + R) + q;
            if (Ln < lsum) {
                const uint32_t lr = LR_EARLY ? lrn[s2] : lrow[Ln];
                ring[s2] = ld_row_v8(a.rows + (static_cast<size_t>(lr & 0x7FFFFFFFu) + sub) * 8);
                hdr[s2] = sub == 0 && (lr >> 31);
            }
        }
        // block sums to smem, unconditionally: a lane past the batch's last
        // line writes into the scratch past it (L < lsum + 8R <= LM + 8R,
        // inside the warp's blk + pad region); the draw forms line sums
        // from the four block sums of a line
#pragma unroll
        for (int s2 = 0; s2 < R; ++s2) blk[4 * (base + 8u * s2 + q) + sub] = bs[s2];
    }
    if (!hooked) at_step2();
}

// The last c in [0, n) with P[c] <= y, for non-decreasing P with P[0] <= y
// (the dense bucket's fp64 chunk / group bases).  4-ary while n > 3: three
// independent probes per level, so about half the dependent shared loads of
// a binary search (the draw is latency-bound); the same c as a binary search.
__device__ __forceinline__ int last_le(const double *P, int n, double y) {
    int c = 0;
#if LDA_DENSE4
    while (n > 3) {
        const int q = n >> 2;
        const int cnt = (P[c + q] <= y) + (P[c + 2 * q] <= y) + (P[c + 3 * q] <= y);
        c += cnt * q;
        n = cnt == 3 ? n - 3 * q : q;
    }
#endif
    while (n > 1) {
        const int h = n >> 1;
        if (P[c + h] <= y) c += h;
        n -= h;
    }
    return c;
}

// Draw of one token of a tile-sampler batch (lane per token, `take` lanes):
// Every search runs on the approximate (monotone) prefixes with plain
// comparisons; the draw is then certified by the margins of the two prefixes
// that bracket x, each against a rigorous bound on its error (the other
// prefixes are farther from x by monotonicity); uncertain -> flag.
template <bool COMPACT = false>
__device__ __forceinline__ void tile_draw(const TileArgs &a, bool take, uint32_t c0, uint32_t nl, uint32_t row,
                                          uint32_t crank, uint64_t cb, double Q64, double gS,
                                          const float *blk, const float *p32, const float *L32, const double *Pc,
                                          int NC, int &z, bool &flag, uint32_t &x0) {
    const int K = a.K;
    const double u = 5.9604644775390625e-08;  // fp32 unit roundoff 2^-24
    z = 0;
    flag = false;
    x0 = 0;
    if (take) {
        double S = 0.0;
#if LDA_LCACHE
        // the prefixes after lines 0..2, kept for the sparse search below
        // (the same doubles it would recompute, in the same order)
        double P0 = 0.0, P1 = 0.0, P2 = 0.0;
        for (uint32_t i = 0; i < nl; ++i) {
            S += f2d_pos(line_sum(blk, c0 + i));
            if (i == 0) P0 = S;
            if (i == 1) P1 = S;
            if (i == 2) P2 = S;
        }
#else
        for (uint32_t i = 0; i < nl; ++i) S += f2d_pos(line_sum(blk, c0 + i));
#endif
        x0 = philox_x0_sched(cb + crank, a.t, a.key0, a.key1);
        const double U = (__hiloint2double(0x43300000, static_cast<int>(x0)) - 4503599627370496.0) *
                         2.3283064365386962890625e-10;  // x0·2^-32, exact
        const double tot = S + Q64;
        const double x = U * tot;
        const double eps = 1.0e-13 * tot * a.slack;  // fp64 roundings of this path
        const double eX = U * gS * S + eps;          // |x' - x|
        const double d = S - x;                       // sparse iff > 0
        const float g32 = static_cast<float>(a.slack);
        if (fabs(d) <= (1.0 - U) * gS * S + eps) {
            flag = true;
        } else if (d > 0.0) {
            // sparse bucket: the line, then the block, whose end prefix first exceeds x
            double C = 0.0, Cn = 0.0;
            uint32_t i = 0;
#if LDA_LCACHE
#if LDA_LSEL
            {
                // branch-free over the first three lines (the common case)
                const bool s0 = P0 > x || nl <= 1, s1 = P1 > x || nl <= 2, s2 = P2 > x || nl <= 3;
                i = s0 ? 0u : s1 ? 1u : s2 ? 2u : 3u;
                C = s0 ? 0.0 : s1 ? P0 : s2 ? P1 : P2;
                Cn = s0 ? P0 : s1 ? P1 : P2;
            }
            if (i == 3) {
                for (;; ++i) {
                    Cn = C + f2d_pos(line_sum(blk, c0 + i));
                    if (Cn > x || i + 1 >= nl) break;
                    C = Cn;
                }
            }
#else
            if (P0 > x || nl <= 1) {
                Cn = P0;
            } else if (P1 > x || nl <= 2) {
                i = 1;
                C = P0;
                Cn = P1;
            } else if (P2 > x || nl <= 3) {
                i = 2;
                C = P1;
                Cn = P2;
            } else {
                C = P2;
                for (i = 3;; ++i) {
                    Cn = C + f2d_pos(line_sum(blk, c0 + i));
                    if (Cn > x || i + 1 >= nl) break;
                    C = Cn;
                }
            }
#endif
#else
            for (;; ++i) {
                Cn = C + f2d_pos(line_sum(blk, c0 + i));
                if (Cn > x || i + 1 >= nl) break;
                C = Cn;
            }
#endif
            const float *bk = blk + 4 * (c0 + i);
            uint32_t b = 0;
#if LDA_BSEL
            {
                // the block: branch-free over the line's first three block-end
                // prefixes (the same doubles as the sequential scan)
                const float4 bq = *reinterpret_cast<const float4 *>(bk);
                const double C1 = C + f2d_pos(bq.x), C2 = C1 + f2d_pos(bq.y), C3 = C2 + f2d_pos(bq.z);
                const bool g1 = C1 > x, g2 = C2 > x, g3 = C3 > x;
                b = g1 ? 0u : g2 ? 1u : g3 ? 2u : 3u;
                const double Cp = g1 ? C : g2 ? C1 : g3 ? C2 : C3;
                Cn = g1 ? C1 : g2 ? C2 : g3 ? C3 : Cn;
                C = Cp;
            }
#else
            for (; b < 3; ++b) {
                const double Cb = C + f2d_pos(bk[b]);
                if (Cb > x) {
                    Cn = Cb;
                    break;
                }
                C = Cb;
            }
#endif
            // certify: C <= x < Cn with margins (C = 0 needs none)
            flag = (x - C <= gS * C + eX && C > 0.0) || (Cn - x <= gS * Cn + eX);
            b += 4 * i;
            // the block's entries in order, relative to r = x - C (fp32):
            // first e with local prefix s_e > r; certify s_{e-1}, s_e
            const float r32 = static_cast<float>(x - C);
            const float eR = static_cast<float>((eX + gS * C + u * (x - C)) * 1.0001 + 1e-30);
            Blk8 w = ld_row_v8(a.rows + (static_cast<size_t>(row) + b) * 8);
            if (b == 0) w.w[0] = 0u;
            float sl = 0.0f, sp = 0.0f, se = 0.0f;
            int ez = -1;
            uint32_t we = 0;
#pragma unroll
            for (int e = 0; e < 8; ++e) {
                const float sn = entry_mass32(w.w[e], p32, sl);
                if (ez < 0 && sn > r32) {
                    ez = e;
                    sp = sl;
                    se = sn;
                    we = w.w[e];
                }
                sl = sn;
            }
            if (ez < 0) {
                flag = true;
            } else {
                flag = flag || (se - r32 <= fmaf(6.2e-7f * g32, se, eR)) ||
                       (sp > 0.0f && r32 - sp <= fmaf(6.2e-7f * g32, sp, eR));   // (2u + 8u)·s
                z = static_cast<int>(we >> kTS);
            }
        } else if (COMPACT) {
            // dense bucket, compact table: the 32-topic group by its fp64 base
            // Pg (Pc here, NC = G groups), then the in-group prefix summed in
            // fp32 from p32 (p32 2u, α u, <= 32 FMA roundings: 35u)
            const double y = U * Q64 - (1.0 - U) * S;
            const double ey = (1.0 - U) * gS * S + eps;
            const int g = last_le(Pc, NC, y);  // last group g with Pg[g] <= y
            const double r = y - Pc[g];
            const float r32 = static_cast<float>(r);
            const float eR = static_cast<float>((ey + u * fabs(r)) * 1.0001 + 1e-30);
            const float a32 = static_cast<float>(a.alpha);
            const int kb = 32 * g, kn = min(K, kb + 32) - kb;
            float l = 0.0f, lp = 0.0f, le = 0.0f;
            int k = -1;
            for (int j = 0; j < kn; ++j) {
                const float ln = fmaf(a32, p32[kb + j], l);
                if (ln > r32) {
                    k = j;
                    lp = l;
                    le = ln;
                    break;
                }
                l = ln;
            }
            if (k < 0) {  // none in the group: the last topic (X6 when it is K-1)
                k = kn - 1;
                z = kb + k;
                flag = z < K - 1 || (k > 0 && r32 - l <= fmaf(2.2e-6f * g32, l, eR));
            } else {
                z = kb + k;
                flag = (z < K - 1 && le - r32 <= fmaf(2.2e-6f * g32, le, eR)) ||
                       (k > 0 && r32 - lp <= fmaf(2.2e-6f * g32, lp, eR)) ||
                       (k == 0 && g > 0 && r <= ey);
            }
        } else {
            // dense bucket: first k with P[k] > y = x - S = U·Q - (1-U)·S;
            // chunk by the fp64 bases Pc, then inside the chunk by L32
            const double y = U * Q64 - (1.0 - U) * S;
            const double ey = (1.0 - U) * gS * S + eps;
            int c = 0;
#if LDA_NC8
            if (NC == 8) {  // K = 1024: two rounds of independent probes instead of three dependent ones
                c = 2 * ((Pc[2] <= y) + (Pc[4] <= y) + (Pc[6] <= y));
                c += Pc[c + 1] <= y;
            } else
#endif
            for (int n = NC; n > 1;) {  // last chunk c with Pc[c] <= y (NC small: binary)
                const int h = n >> 1;
                if (Pc[c + h] <= y) c += h;
                n -= h;
            }
            const double r = y - Pc[c];
            const float r32 = static_cast<float>(r);
            const float eR = static_cast<float>((ey + u * fabs(r)) * 1.0001 + 1e-30);
            const int kb = 128 * c, kn = min(K, kb + 128) - kb;
            int k = 0;  // first k in the chunk with L32 > r (kn - 1 if none)
#if LDA_DENSE4
            if (kn == 128) {
                // 4-ary: three independent probes per level (4 dependent
                // shared loads instead of 7).  Same k when L32 is monotone;
                // any other k fails the bracket certification below.
#pragma unroll
                for (int g = 32; g >= 2; g >>= 2) {
                    const float a0 = L32[l32_idx(kb + k + g - 1)], a1 = L32[l32_idx(kb + k + 2 * g - 1)];
                    const float a2 = L32[l32_idx(kb + k + 3 * g - 1)];
                    k += g * ((a0 <= r32) + (a1 <= r32) + (a2 <= r32));
                }
                if (L32[l32_idx(kb + k)] <= r32) k += 1;
            } else
#endif
            for (int n = kn; n > 1;) {
                const int h = n >> 1;
                if (L32[l32_idx(kb + k + h - 1)] <= r32) k += h;
                n -= h;
            }
            z = kb + k;
            // certify the bracket: L[z-1] <= y < L[z] (Pc[c] when k = 0)
            const float le = L32[l32_idx(z)], lp = k > 0 ? L32[l32_idx(z - 1)] : 0.0f;
            flag = (z < K - 1 && le - r32 <= fmaf(1.3e-7f * g32, le, eR)) ||
                   (k > 0 && r32 - lp <= fmaf(1.3e-7f * g32, lp, eR)) ||
                   (k == 0 && c > 0 && r <= ey);
        }
    }
}

// Exact fp64 redraw of a batch's uncertain tokens (one at a time by the
// warp), then z and the fused recount (ϕ update, L1273-1285).
__device__ __forceinline__ void tile_finish(const TileArgs &a, bool take, bool flag, int z, uint32_t row,
                                            uint32_t nnz, uint32_t x0, uint32_t p, const int32_t *nwk_row,
                                            int32_t *row_next, int *nkh, const double *B, int G, int gsz,
                                            unsigned &n_exact) {
    // nkh: the n_k histogram -- the CTA's in shared memory, or the global
    // next n_k (the large-K kernel keeps its shared memory for warps)
    const int lane = threadIdx.x & 31;
    const int K = a.K;
    // ---- exact fp64 redraw of the uncertain tokens, one at a time by the warp
    unsigned fl = __ballot_sync(kFull, flag);
    while (fl) {
        const int f = __ffs(fl) - 1;
        fl &= fl - 1;
        const uint32_t rf = __shfl_sync(kFull, row, f);
        const uint32_t nf = __shfl_sync(kFull, nnz, f);
        const uint32_t xf = __shfl_sync(kFull, x0, f);
        const int zf = draw_exact_warp(nwk_row, a.denom, a.rows + static_cast<size_t>(rf) * 8, nf, xf, K,
                                       a.alpha, a.beta, B, G, gsz);
        if (lane == f) z = zf;
        ++n_exact;
    }
    // ---- z and the fused recount
    if (take) {
        a.z[p] = static_cast<uint16_t>(z);
    }
    if (take && a.recount) {
        const unsigned act = __activemask();
        const unsigned peers = __match_any_sync(act, z);
        if (lane == __ffs(peers) - 1) {
            const int c = __popc(peers);
            atomicAdd(row_next + z, c);
            atomicAdd(&nkh[z], c);
        }
    }
    __syncwarp();
}

template <int R>
__global__ void __launch_bounds__(32 * LDA_TILE_WPC, LDA_TILE_MINB) sweep_tile_kernel(TileArgs a) {
    extern __shared__ double smem_dd[];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int K = a.K;
    const int K4 = (K + 3) & ~3;
    const int NC = (K + 127) / 128;
    const int LM = a.lmax;
    int *nkh = reinterpret_cast<int *>(smem_dd);
    char *wb = reinterpret_cast<char *>(nkh + K4) + static_cast<size_t>(warp) * tile_warp_bytes(K, LM);
    double *Pc = reinterpret_cast<double *>(wb);
    float *p32 = reinterpret_cast<float *>(Pc + tab_nc2(K));
    float *L32 = p32 + K4;
    float *blk = L32 + 128 * NC;           // 4 block sums per line
    // blk: 4 block sums per line; the next LM floats pad it for the walk's
    // unconditional stores past the batch's last line (LM >= 8R)
    uint32_t *lrow = reinterpret_cast<uint32_t *>(blk + 5 * LM);
    uint32_t *tcum = lrow + LM;
    uint64_t *bar = reinterpret_cast<uint64_t *>(tcum + 32);
    for (int k = threadIdx.x; k < K; k += blockDim.x) nkh[k] = 0;
    if (lane == 0) mbar_init(bar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    __syncthreads();
    unsigned n_exact = 0;
    int cur_word = -1;
    uint32_t phase = 0;
#if LDA_TILE_STATS
    unsigned long long st_batches = 0, st_tokens = 0, st_lines = 0, st_rows = 0, st_steps = 0;
#endif
    const double u = 5.9604644775390625e-08;  // fp32 unit roundoff 2^-24
    // rounding bound of every prefix of the walk: p32 2u + 4-FFMA chain + 1
    // (block sum) + 2 (quad line sum), accumulated in fp64
    const double gS = 9.5 * u * a.slack;

    auto claim = [&]() {
        uint32_t c = 0;
        if (lane == 0) c = atomicAdd(a.counter, 1u);
        return __shfl_sync(kFull, c, 0);
    };
    const TileItem none = {0u, 0u, 0u, 0u};
    uint32_t ci = claim();
    if (ci >= a.n_items) ci = 0xFFFFFFFFu;
    TileItem it = ci != 0xFFFFFFFFu ? a.items[ci] : none;
    uint32_t cn = ci != 0xFFFFFFFFu ? claim() : 0xFFFFFFFFu;
    TileItem itn = cn < a.n_items ? a.items[cn] : none;
    if (lane == 0 && cn < a.n_items && itn.word != it.word)
        prefetch_l2_table(a.wtab + static_cast<size_t>(itn.word) * a.wt_bytes, a.wt_bytes);
    // Batch head (up to 32 tokens whose θ rows have at most LM lines in
    // total; consecutive tokens of one document -- a (word, doc) pair --
    // share the walk of its row): line table in smem, first R lines of the
    // walk in flight.  Built for the next batch before the current batch's
    // draw, so that its loads overlap the draw.
    Blk8 ring[R];
    bool hdr[R];  // the line in ring slot s2 is the first of its row (word 0 = nnz header)
    auto head = [&](uint32_t row, uint32_t nnz, bool valid) {
        return tile_head<R>(a, row, nnz, valid, LM, lrow, ring, hdr);
    };
    // the first batch
    uint32_t row = 0, crank = 0, nnz = 0;
    if (lane < it.n) {
        row = ld_stream_u32(a.tok_row + it.pos + lane);
        crank = it.crank0 + lane;
        nnz = ld_row_u32(a.rows + static_cast<size_t>(row) * 8);
    }
    TileHead hd = head(row, nnz, static_cast<uint32_t>(lane) < it.n);
    uint32_t b0 = 0;
    bool new_item = true;
    const int32_t *nwk_row = nullptr;
    int32_t *row_next = nullptr;
    uint64_t cb = 0;
    double Q64 = 0.0;
    while (ci != 0xFFFFFFFFu) {
        if (new_item) {
            if (static_cast<int>(it.word) != cur_word) {
                // the word's table -> smem by one bulk copy (all lanes are past their last read)
                __syncwarp();
                if (lane == 0) {
                    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                    mbar_arrive_expect_tx(bar, a.wt_bytes);
                    bulk_g2s(Pc, a.wtab + static_cast<size_t>(it.word) * a.wt_bytes, a.wt_bytes, bar);
                }
                mbar_wait(bar, phase);
                phase ^= 1u;
                cur_word = static_cast<int>(it.word);
            }
            Q64 = Pc[NC];
            cb = __ldg(a.cbase + it.word);
            nwk_row = a.nwk + static_cast<size_t>(it.word) * K;
            row_next = a.nwk_next + static_cast<size_t>(it.word) * K;
            new_item = false;
        }
        // ---- this batch
        const uint32_t p = it.pos + b0 + lane;
        const bool take = hd.take;
#if LDA_TILE_STATS
        {
            const unsigned nd = __popc(__ballot_sync(kFull, take && !hd.dup));
            if (lane == 0) {
                st_batches += 1;
                st_tokens += hd.nb;
                st_lines += hd.lsum;
                st_rows += nd;
                st_steps += (hd.lsum + 8u * LDA_TRING - 1) / (8u * LDA_TRING);
            }
        }
#endif
        const int nb = hd.nb;
        const uint32_t lsum = hd.lsum, c0 = hd.c0, nl = hd.nl;
        // ---- the next batch: this item's next tokens, else the next item's first
        const uint32_t b1 = b0 + static_cast<uint32_t>(nb);
        const bool more = b1 < it.n;
        const uint32_t nxt_pos = more ? it.pos + b1 : itn.pos;
        const uint32_t nxt_n = more ? it.n - b1 : (cn < a.n_items ? itn.n : 0u);
        const bool nxt_valid = static_cast<uint32_t>(lane) < nxt_n;
        uint32_t n_row = 0, n_nnz = 0;
        const uint32_t n_crank = (more ? it.crank0 + b1 : itn.crank0) + lane;
        if (nxt_valid) n_row = ld_stream_u32(a.tok_row + nxt_pos + lane);
        // ---- walk (the next batch's row headers issued after its first step)
        tile_walk<R>(a, lsum, lrow, ring, hdr, p32, blk, [&] {
            if (nxt_valid) n_nnz = ld_row_u32(a.rows + static_cast<size_t>(n_row) * 8);
        });
        __syncwarp();
        // ---- the next batch's head: its line table and first lines, in flight during this draw
        const TileHead hn = head(n_row, n_nnz, nxt_valid);

        // ---- draw: lane per token (lanes < nb).  Every search below runs on
        // the approximate (monotone) prefixes with plain comparisons; the
        // draw is then certified by the margins of the two prefixes that
        // bracket x, each against a rigorous bound on its error (the other
        // prefixes are farther from x by monotonicity); uncertain -> flag.
        int z;
        bool flag;
        uint32_t x0;
        tile_draw(a, take, c0, nl, row, crank, cb, Q64, gS, blk, p32, L32, Pc, NC, z, flag, x0);
        tile_finish(a, take, flag, z, row, nnz, x0, p, nwk_row, row_next, nkh, Pc, NC, 128, n_exact);
        // ---- advance
        row = n_row;
        crank = n_crank;
        nnz = n_nnz;
        hd = hn;
        if (more) {
            b0 = b1;
        } else {
            ci = cn < a.n_items ? cn : 0xFFFFFFFFu;
            if (ci == 0xFFFFFFFFu) break;
            it = itn;
            b0 = 0;
            new_item = true;
            cn = claim();
            itn = cn < a.n_items ? a.items[cn] : none;
            if (lane == 0 && cn < a.n_items && itn.word != it.word)
                prefetch_l2_table(a.wtab + static_cast<size_t>(itn.word) * a.wt_bytes, a.wt_bytes);
        }
    }
    __syncthreads();
    if (a.recount)
        for (int k = threadIdx.x; k < K; k += blockDim.x)
            if (nkh[k]) atomicAdd(a.nk_next + k, nkh[k]);
    if (a.n_exact && lane == 0 && n_exact) atomicAdd(a.n_exact, static_cast<unsigned long long>(n_exact));
#if LDA_TILE_STATS
    if (lane == 0) {
        atomicAdd(&g_tile_stats[0], st_batches);
        atomicAdd(&g_tile_stats[1], st_tokens);
        atomicAdd(&g_tile_stats[2], st_lines);
        atomicAdd(&g_tile_stats[3], st_rows);
        atomicAdd(&g_tile_stats[4], st_steps);
    }
#endif
}


// ---------------------------------------------------------------------------
// a3 + a4, tile sampler for large K (sampler 3): the 8 warps of a CTA share
// the word table, double-buffered in shared memory -- at K = 8192 a per-warp
// table (66 KB) would leave 2-3 warps per SM.  The CTA takes the work items
// in queue order; its warps claim 32-token slots of the current item and walk
// / draw them exactly as sweep_tile_kernel does (same helpers, same
// certification); the last warp to leave an item refills that buffer with
// the CTA's next item (bulk copy), while the other warps already work on the
// item in the other buffer.
// ---------------------------------------------------------------------------
__host__ __device__ constexpr size_t tile_cta_warp_bytes(int lmax) {
    return static_cast<size_t>(lmax) * (16 + 4 + 4) + 32 * 4 + 16;
}
// large K (gnk): compact tables and n_k by global reductions; nb table buffers (<= 4)
__host__ __device__ constexpr size_t tile_cta_bytes(int K, int lmax, int nwarps, bool gnk, int nb) {
    return (gnk ? 0 : static_cast<size_t>(4) * ((K + 3) & ~3)) +
           static_cast<size_t>(nb) * (gnk ? tab_bytes_compact(K) : tab_bytes(K)) +
           nwarps * tile_cta_warp_bytes(lmax) + 256;
}

__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

// GNK: n_k by warp-aggregated global reductions (large K: the shared memory
// goes to warps); else a per-CTA shared histogram (global reductions on few
// addresses contend at small K).
template <int R, bool GNK>
__global__ void __launch_bounds__(512, 1) sweep_tile_cta_kernel(TileArgs a) {
    extern __shared__ double smem_dd[];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nwarps = blockDim.x >> 5;
    const int K = a.K;
    const int K4 = (K + 3) & ~3;
    const int NC = GNK ? (K + 31) / 32 : (K + 127) / 128;  // groups of the dense prefix's fp64 level
    const int LM = a.lmax;
    const int NB = a.nbuf;  // table buffers (2..4): items in flight per CTA
    const size_t wt = a.wt_bytes;
    int *nkh = GNK ? a.nk_next : reinterpret_cast<int *>(smem_dd);
    char *tabs = reinterpret_cast<char *>(smem_dd) + (GNK ? 0 : 4 * K4);
    char *wb = tabs + NB * wt + static_cast<size_t>(warp) * tile_cta_warp_bytes(LM);
    float *blk = reinterpret_cast<float *>(wb);
    uint32_t *lrow = reinterpret_cast<uint32_t *>(blk + 5 * LM);  // blk + pad (see sweep_tile_kernel)
    char *ctrl = tabs + NB * wt + static_cast<size_t>(nwarps) * tile_cta_warp_bytes(LM);
    uint64_t *bar = reinterpret_cast<uint64_t *>(ctrl);         // [4]
    TileItem *items = reinterpret_cast<TileItem *>(ctrl + 32);  // [4]
    uint32_t *slot = reinterpret_cast<uint32_t *>(ctrl + 96);   // [4]
    uint32_t *left = slot + 4;                                  // [4]
    int *bsw = reinterpret_cast<int *>(ctrl + 128);             // [4] f2: the sparse word whose p32 row the
                                                                //     buffer holds (-1: a dense table / none)
    const double gS = 9.5 * 5.9604644775390625e-08 * a.slack;
    const int K4c = (K + 3) & ~3;
    const uint32_t pg_bytes = static_cast<uint32_t>(8 * tab_g2(K));

    // buffer b <- the CTA's next work item (its table by bulk copy); the end
    // of the queue is an item with n = 0.  items[b] / slot[b] / left[b] are
    // published to the other warps by the buffer's mbarrier: the arrive below
    // has release semantics and their try_wait acquire semantics (CTA scope);
    // compute-sanitizer's racecheck does not model mbarrier ordering and
    // reports this handoff as a hazard (memcheck is clean).  The loader runs
    // only after every warp has left the buffer (left[b] reached 0).
    // Run by a whole warp.  A sparse word (f2) is built in place by the warp:
    // its Pg copied, the p32 row = the smoothing row s32 (copied in full when
    // the buffer held a dense table, else restored at the previous sparse
    // word's topics) patched at the word's nonzero topics; plain smem stores,
    // published by the warp's arrive.  Dense tables: one bulk copy.
    auto load = [&](int b) {
        uint32_t ci = 0;
        if (lane == 0) ci = atomicAdd(a.counter, 1u);
        ci = __shfl_sync(kFull, ci, 0);
        TileItem it = {0u, 0u, 0u, 0u};
        if (ci < a.n_items) it = a.items[ci];
        uint32_t o0 = 0, o1 = 0;
        if (GNK && a.sp_off && it.n) {
            o0 = __ldg(a.sp_off + it.word);
            o1 = __ldg(a.sp_off + it.word + 1);
        }
        const int prev = bsw[b];
        __syncwarp();
        if (lane == 0) {
            items[b] = it;
            slot[b] = 0u;
            left[b] = static_cast<uint32_t>(nwarps);
            bsw[b] = o1 > o0 ? static_cast<int>(it.word) : -1;
        }
        if (o1 > o0) {
            char *tb = tabs + b * wt;
            float *p32s = reinterpret_cast<float *>(tb + pg_bytes);
            if (prev < 0) {
                for (int i = lane; i < K4c / 4; i += 32)
                    reinterpret_cast<float4 *>(p32s)[i] = __ldg(reinterpret_cast<const float4 *>(a.s32) + i);
            } else {
                const uint32_t *pe = a.sp_ent + 2 * static_cast<size_t>(__ldg(a.sp_off + prev));
                const uint32_t pn = __ldg(a.sp_nnz + prev);
                for (uint32_t j = lane; j < pn; j += 32) {
                    const uint32_t t = __ldg(pe + 2 * j);
                    p32s[t] = __ldg(a.s32 + t);
                }
            }
            const double2 *src = reinterpret_cast<const double2 *>(a.wtab + static_cast<size_t>(it.word) * a.wt_bytes);
            for (uint32_t i = lane; i < pg_bytes / 16; i += 32) reinterpret_cast<double2 *>(tb)[i] = __ldg(src + i);
            __syncwarp();
            const uint2 *e2 = reinterpret_cast<const uint2 *>(a.sp_ent) + o0;
            const uint32_t n = __ldg(a.sp_nnz + it.word);
            for (uint32_t j = lane; j < n; j += 32) {
                const uint2 e = __ldg(e2 + j);
                p32s[e.x] = __uint_as_float(e.y);
            }
            __syncwarp();
            __threadfence_block();
            if (lane == 0) mbar_arrive(bar + b);
        } else {
            // the buffer's previous contents were written by this warp's or
            // other warps' generic stores (a sparse word) or read by them
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            __syncwarp();
            if (lane == 0) {
                if (it.n) {
                    mbar_arrive_expect_tx(bar + b, a.wt_bytes);
                    bulk_g2s(tabs + b * wt, a.wtab + static_cast<size_t>(it.word) * a.wt_bytes, a.wt_bytes, bar + b);
                } else {
                    mbar_arrive(bar + b);
                }
            }
        }
    };
    if (!GNK)
        for (int k = threadIdx.x; k < K; k += blockDim.x) nkh[k] = 0;
    if (threadIdx.x == 0) {
        for (int b = 0; b < NB; ++b) {
            mbar_init(bar + b, 1);
            bsw[b] = -1;
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 0) {
        __syncwarp();
        for (int b = 0; b < NB; ++b) load(b);
    }
    __syncthreads();

    unsigned n_exact = 0;
    uint32_t phases = 0u;  // bit b: the parity of buffer b's next completion
    Blk8 ring[R];
    bool hdr[R];
    for (int b = 0;; b = b + 1 < NB ? b + 1 : 0) {
        mbar_wait(bar + b, (phases >> b) & 1u);
        phases ^= 1u << b;
        const TileItem it = items[b];
        if (it.n == 0) break;
        const double *Pc = reinterpret_cast<const double *>(tabs + b * wt);
        const float *p32 = reinterpret_cast<const float *>(Pc + (GNK ? tab_g2(K) : tab_nc2(K)));
        const float *L32 = p32 + K4;
        const double Q64 = Pc[NC];
        const uint64_t cb = __ldg(a.cbase + it.word);
        const int32_t *nwk_row = a.nwk + static_cast<size_t>(it.word) * K;
        int32_t *row_next = a.nwk_next + static_cast<size_t>(it.word) * K;
        for (;;) {
            uint32_t sl = 0;
            if (lane == 0) sl = atomicAdd(slot + b, 1u);
            sl = __shfl_sync(kFull, sl, 0);
            if (32u * sl >= it.n) break;
            const uint32_t t1 = min(it.n, 32u * sl + 32u);
            for (uint32_t b0 = 32u * sl; b0 < t1;) {
                const bool valid = b0 + lane < t1;
                const uint32_t p = it.pos + b0 + lane;
                uint32_t row = 0, crank = 0, nnz = 0;
                if (valid) {
                    row = ld_stream_u32(a.tok_row + p);
                    crank = it.crank0 + b0 + lane;
                    nnz = ld_row_u32(a.rows + static_cast<size_t>(row) * 8);
                }
                const TileHead hd = tile_head<R>(a, row, nnz, valid, LM, lrow, ring, hdr);
                tile_walk<R, GNK>(a, hd.lsum, lrow, ring, hdr, p32, blk, [] {});
                __syncwarp();
                int z;
                bool flag;
                uint32_t x0;
                tile_draw<GNK>(a, hd.take, hd.c0, hd.nl, row, crank, cb, Q64, gS, blk, p32, L32, Pc, NC, z,
                               flag, x0);
                tile_finish(a, hd.take, flag, z, row, nnz, x0, p, nwk_row, row_next, nkh, Pc, NC, GNK ? 32 : 128,
                            n_exact);
                b0 += static_cast<uint32_t>(hd.nb);
            }
        }
        // leave the item; the last warp out refills the buffer
        __syncwarp();
        __threadfence_block();
        uint32_t was = 0;
        if (lane == 0) was = atomicSub(left + b, 1u);
        was = __shfl_sync(kFull, was, 0);
        if (was == 1u) {
            __threadfence_block();
            load(b);
        }
    }
    if (!GNK) {
        __syncthreads();
        if (a.recount)
            for (int k = threadIdx.x; k < K; k += blockDim.x)
                if (nkh[k]) atomicAdd(a.nk_next + k, nkh[k]);
    }
    if (a.n_exact && lane == 0 && n_exact) atomicAdd(a.n_exact, static_cast<unsigned long long>(n_exact));
}

// ---------------------------------------------------------------------------
// a4 epilogue (separate kernel): n_wk / n_k recount from z.
// ---------------------------------------------------------------------------
// a0 on the device: the θ row of every token's document at its word-major
// position (warp per document: coalesced doc_map reads, scattered stores).
// One warp per document and no grid-stride loop: the blocks in flight are
// consecutive documents, so the scattered stores stay inside one tile's part
// of the word-major stream (L2).
__global__ void tok_row_kernel(const uint32_t *__restrict__ doc_ptr32, const uint32_t *__restrict__ row_off32,
                               const uint32_t *__restrict__ doc_map, uint32_t *__restrict__ tok_row, int64_t D) {
    const int lane = threadIdx.x & 31;
    {
        const int64_t d = static_cast<int64_t>(blockIdx.x) * (blockDim.x >> 5) + (threadIdx.x >> 5);
        if (d >= D) return;
        const uint32_t s = doc_ptr32[d], e = doc_ptr32[d + 1], row = row_off32[d];
        for (uint32_t i = s + lane; i < e; i += 32) tok_row[doc_map[i]] = row;
    }
}

__global__ void zero_rows_kernel(const int32_t *__restrict__ words, int64_t n, int32_t *__restrict__ nwk,
                                 int K) {
    for (int64_t i = blockIdx.x; i < n; i += gridDim.x) {
        int32_t *row = nwk + static_cast<size_t>(words[i]) * K;
        for (int k = threadIdx.x; k < K; k += blockDim.x) row[k] = 0;
    }
}

// Segmented recount (the ϕ update as a separate pass, L1273-1285): per work
// item (a word's virtual token range, <= recount_tokens) a CTA builds the
// topic histogram in shared memory, the warps taking the word's runs in turn
// (each run contiguous in the word-major stream: coalesced z reads, no
// per-token search), then writes the word's row of n_wk (global atomics only
// for words split over several items) and accumulates n_k.
// GMEM (K > 16384): the CTA's two K-length histograms in a global scratch
// slice (zero on entry, left zero on exit) instead of shared memory.
template <bool GMEM>
__global__ void recount_kernel(const RecountChunk *__restrict__ rc, int64_t n_rc,
                               const Seg *__restrict__ segs, int K, const uint16_t *__restrict__ z,
                               int32_t *__restrict__ nwk, int32_t *__restrict__ nk,
                               uint32_t *__restrict__ counter, int *__restrict__ gscratch) {
    extern __shared__ int smem_i[];
    int *hist = GMEM ? gscratch + static_cast<size_t>(blockIdx.x) * 2 * K : smem_i, *nkp = hist + K;
    __shared__ int s_ci;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nwarps = blockDim.x >> 5;
    if (!GMEM)
        for (int k = threadIdx.x; k < 2 * K; k += blockDim.x) smem_i[k] = 0;
    __syncthreads();
    for (;;) {
        if (threadIdx.x == 0) s_ci = static_cast<int>(atomicAdd(counter, 1u));
        __syncthreads();
        const int ci = s_ci;
        if (ci >= n_rc) break;
        const RecountChunk c = rc[ci];
        const uint32_t w = c.word & 0x7FFFFFFFu;
        const bool split = (c.word >> 31) != 0u;
        const uint32_t vb = c.vbegin, ve = c.vbegin + c.vcount;
        // runs s = seg0 + warp, seg0 + warp + nwarps, ... while they start before ve
        for (uint32_t si = c.seg0 + warp; si < c.segN; si += nwarps) {
            const Seg sg = segs[si];
            if (sg.vstart >= ve) break;
            const uint32_t rv0 = max(sg.vstart, vb), rv1 = min(segs[si + 1].vstart, ve);
            const uint32_t p0 = sg.pos + (rv0 - sg.vstart);
            for (uint32_t v = rv0 + lane; v < rv1; v += 32) atomicAdd(&hist[z[p0 + (v - rv0)]], 1);
        }
        __syncthreads();
        int32_t *row = nwk + static_cast<size_t>(w) * K;
        for (int k = threadIdx.x; k < K; k += blockDim.x) {
            const int h = hist[k];
            if (split) {
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
        if (nkp[k]) {
            atomicAdd(nk + k, nkp[k]);
            if (GMEM) nkp[k] = 0;
        }
}

// ---------------------------------------------------------------------------
// a5: θ rebuild.  One warp per document: gather z through the doc-word map,
// count topics in a per-warp shared histogram + bitmap, then write the row
// as ascending (topic << 18 | count) entries with a popc scan over the bitmap.
// O(L_d + K/32) per document instead of the paper's dense O(K) row.
// ---------------------------------------------------------------------------
// Two-phase variant, phase A: z in document order, zd[i] = z[doc_map[i]]
// (independent gathers with high memory-level parallelism, in doc order).
__global__ void gather_z_kernel(const uint32_t *__restrict__ doc_map, const uint16_t *__restrict__ z,
                                uint16_t *__restrict__ zd, int64_t T) {
    // 8 independent gathers per thread (two 16-byte reads of the map)
    const int64_t i0 = (static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x) * 8;
    if (i0 + 7 < T) {
        const uint4 m0 = __ldcs(reinterpret_cast<const uint4 *>(doc_map + i0));
        const uint4 m1 = __ldcs(reinterpret_cast<const uint4 *>(doc_map + i0 + 4));
        const uint16_t a0 = z[m0.x], a1 = z[m0.y], a2 = z[m0.z], a3 = z[m0.w];
        const uint16_t a4 = z[m1.x], a5 = z[m1.y], a6 = z[m1.z], a7 = z[m1.w];
        uint4 o;
        o.x = a0 | (static_cast<uint32_t>(a1) << 16);
        o.y = a2 | (static_cast<uint32_t>(a3) << 16);
        o.z = a4 | (static_cast<uint32_t>(a5) << 16);
        o.w = a6 | (static_cast<uint32_t>(a7) << 16);
        __stcs(reinterpret_cast<uint4 *>(zd + i0), o);
    } else {
        for (int64_t i = i0; i < T; ++i) zd[i] = z[doc_map[i]];
    }
}

// z in document order -> word-major (lda_set_z): zw[doc_map[i]] = zd[i]
__global__ void scatter_z_kernel(const uint32_t *__restrict__ doc_map, const uint16_t *__restrict__ zd,
                                 uint16_t *__restrict__ zw, int64_t T) {
    for (int64_t i = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x; i < T;
         i += static_cast<int64_t>(gridDim.x) * blockDim.x)
        zw[doc_map[i]] = zd[i];
}

// Phase B: zd is z in document order (gather_z_kernel).
// GMEM (K > 16384): the warp's histogram + bitmap in a global scratch slice
// (zero on entry, left zero) instead of shared memory; TS: entry shift.
template <bool GMEM, int TS>
__global__ void theta_kernel(const uint32_t *__restrict__ doc_ptr32, const uint32_t *__restrict__ row_off32,
                             const uint16_t *__restrict__ zd,
                             uint32_t *__restrict__ rows, int64_t D, int K,
                             unsigned long long *__restrict__ stat, uint32_t *__restrict__ gscratch) {
    extern __shared__ uint32_t smem_u[];
    const int Kw = (K + 31) >> 5;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, wpb = blockDim.x >> 5;
    uint32_t *cnt = (GMEM ? gscratch + static_cast<size_t>(blockIdx.x) * wpb * (K + Kw) : smem_u) +
                    static_cast<size_t>(warp) * (K + Kw);
    uint32_t *bits = cnt + K;
    if (!GMEM)
        for (int k = lane; k < K + Kw; k += 32) cnt[k] = 0u;
    __syncwarp();
    unsigned long long s_lnnz = 0, s_nnz = 0;
    const int64_t nw = static_cast<int64_t>(gridDim.x) * wpb;
    int64_t d = static_cast<int64_t>(blockIdx.x) * wpb + warp;
    // the next document's bounds and row, loaded one document ahead
    uint32_t n_s = 0, n_e = 0, n_off = 0;
    if (d < D) {
        n_s = doc_ptr32[d];
        n_e = doc_ptr32[d + 1];
        n_off = row_off32[d];
    }
    for (; d < D; d += nw) {
        const uint32_t s = n_s, e = n_e;
        uint32_t *row = rows + static_cast<size_t>(n_off) * 8;
        const uint32_t old_nnz = row[0];  // issued early: its latency overlaps the histogram
        if (d + nw < D) {
            n_s = doc_ptr32[d + nw];
            n_e = doc_ptr32[d + nw + 1];
            n_off = row_off32[d + nw];
        }
        // up to 4 topics per lane in flight, then the shared histogram
        for (uint32_t i0 = s; i0 < e; i0 += 128) {
            uint32_t kk[4];
#pragma unroll
            for (int r = 0; r < 4; ++r) {
                const uint32_t i = i0 + 32u * r + lane;
                kk[r] = i < e ? zd[i] : 0xFFFFFFFFu;
            }
#pragma unroll
            for (int r = 0; r < 4; ++r) {
                if (kk[r] != 0xFFFFFFFFu) {
                    atomicAdd(&cnt[kk[r]], 1u);
                    atomicOr(&bits[kk[r] >> 5], 1u << (kk[r] & 31));
                }
            }
        }
        __syncwarp();
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
                row[1 + pos++] = (k << TS) | cnt[k];
                cnt[k] = 0u;
            }
            if (qq < Kw) bits[qq] = 0u;
            base += __shfl_sync(kFull, incl, 31);
        }
        // words past the new last entry that held entries before are zeroed:
        // every word of the row past 1 + nnz stays zero (rows start zeroed)
        for (uint32_t i = 1u + base + lane; i < 1u + old_nnz; i += 32u) row[i] = 0u;
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

__global__ void ll_doc_kernel(const uint32_t *__restrict__ doc_ptr32, const uint32_t *__restrict__ row_off32,
                              const uint32_t *__restrict__ rows, int64_t D, double alpha, double lga,
                              double Kalpha, double lgKa, double *__restrict__ part) {
    __shared__ double sh[32];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, wpb = blockDim.x >> 5;
    double s = 0.0;
    const int64_t nw = static_cast<int64_t>(gridDim.x) * wpb;
    for (int64_t d = static_cast<int64_t>(blockIdx.x) * wpb + warp; d < D; d += nw) {
        const uint32_t *row = rows + static_cast<size_t>(row_off32[d]) * 8;
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
// Peer-memory collectives (the in-process PeerComm backend of Eq. 4's
// exchange, comm.cpp): every rank's buffer is a device pointer readable by
// the others (the same GPU, or P2P over NVLink).  16-byte vectors, L2-only
// loads (another GPU's memory is never cached in this SM's L1).
// ---------------------------------------------------------------------------
struct PeerPtrs {
    const char *p[kMaxPeers];
};

__host__ __device__ inline size_t peer_slice_lo(size_t n, int world, int q, size_t vw) {
    return q >= world ? n : (n * static_cast<size_t>(q) / static_cast<size_t>(world)) / vw * vw;
}

template <class T>
__global__ void peer_rs_kernel(const __grid_constant__ PeerPtrs src, int world, T *__restrict__ own, size_t lo,
                               size_t hi) {
    constexpr int VW = 16 / sizeof(T);
    const size_t nv = (hi - lo) / VW;
    const size_t stride = static_cast<size_t>(gridDim.x) * blockDim.x;
    for (size_t i = static_cast<size_t>(blockIdx.x) * blockDim.x + threadIdx.x; i < nv; i += stride) {
        const size_t off = (lo + i * VW) * sizeof(T);
        T acc[VW];
#pragma unroll
        for (int j = 0; j < VW; ++j) acc[j] = T(0);
        for (int q = 0; q < world; ++q) {
            const uint4 v = __ldcg(reinterpret_cast<const uint4 *>(src.p[q] + off));
            T t[VW];
            memcpy(t, &v, 16);
#pragma unroll
            for (int j = 0; j < VW; ++j) acc[j] += t[j];
        }
        uint4 o;
        memcpy(&o, acc, 16);
        *reinterpret_cast<uint4 *>(reinterpret_cast<char *>(own) + off) = o;
    }
    // ragged tail of the last slice
    for (size_t e = lo + nv * VW + static_cast<size_t>(blockIdx.x) * blockDim.x + threadIdx.x; e < hi; e += stride) {
        T acc = T(0);
        for (int q = 0; q < world; ++q) acc += reinterpret_cast<const T *>(src.p[q])[e];
        own[e] = acc;
    }
}

__global__ void peer_copy_kernel(const char *__restrict__ src, char *__restrict__ dst, size_t b0, size_t b1) {
    // [b0, b1) bytes, b0 16-byte aligned
    const size_t nv = (b1 - b0) / 16;
    const size_t stride = static_cast<size_t>(gridDim.x) * blockDim.x;
    for (size_t i = static_cast<size_t>(blockIdx.x) * blockDim.x + threadIdx.x; i < nv; i += stride)
        *reinterpret_cast<uint4 *>(dst + b0 + 16 * i) = __ldcg(reinterpret_cast<const uint4 *>(src + b0 + 16 * i));
    for (size_t b = b0 + 16 * nv + static_cast<size_t>(blockIdx.x) * blockDim.x + threadIdx.x; b < b1; b += stride)
        dst[b] = src[b];
}

static unsigned peer_grid(size_t work) {
    const size_t g = (work + 255) / 256;
    return static_cast<unsigned>(std::max<size_t>(1, std::min<size_t>(g, 148 * 8)));
}

int launch_peer_reduce_scatter(void *const *ptrs, int world, int rank, void *own, size_t n, size_t esz, int is_f64,
                               void *stream) {
    if (world < 1 || world > kMaxPeers) return cudaErrorInvalidValue;
    PeerPtrs pp{};
    for (int q = 0; q < world; ++q) pp.p[q] = static_cast<const char *>(ptrs[q]);
    const size_t vw = 16 / esz;
    const size_t lo = peer_slice_lo(n, world, rank, vw), hi = peer_slice_lo(n, world, rank + 1, vw);
    if (hi <= lo) return cudaSuccess;
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    if (is_f64)
        peer_rs_kernel<double><<<peer_grid((hi - lo) / vw + 1), 256, 0, st>>>(pp, world, static_cast<double *>(own),
                                                                            lo, hi);
    else
        peer_rs_kernel<int32_t><<<peer_grid((hi - lo) / vw + 1), 256, 0, st>>>(pp, world,
                                                                             static_cast<int32_t *>(own), lo, hi);
    return cudaGetLastError();
}

int launch_peer_all_gather(void *const *ptrs, int world, int rank, void *own, size_t n, size_t esz, void *stream) {
    if (world < 1 || world > kMaxPeers) return cudaErrorInvalidValue;
    const size_t vw = 16 / esz;
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    for (int q = 0; q < world; ++q) {
        if (q == rank) continue;
        const size_t lo = peer_slice_lo(n, world, q, vw), hi = peer_slice_lo(n, world, q + 1, vw);
        if (hi <= lo) continue;
        peer_copy_kernel<<<peer_grid((hi - lo) / vw + 1), 256, 0, st>>>(static_cast<const char *>(ptrs[q]),
                                                                       static_cast<char *>(own), lo * esz, hi * esz);
    }
    return cudaGetLastError();
}

// ---------------------------------------------------------------------------
// Launchers
// ---------------------------------------------------------------------------
int configure_kernels(DevState &s) {
    cudaError_t e;
    const void *sampler0_fn = nullptr;
    int dev = 0;
    if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
    if ((e = cudaDeviceGetAttribute(&s.num_sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess) return e;
    int max_optin = 0;
    if ((e = cudaDeviceGetAttribute(&max_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev)) != cudaSuccess)
        return e;
    // sampler: p*/P (+ fused-recount histograms) in smem when they fit
    {
        const size_t blk = sizeof(double) * kMaxBlk * kSweepThreads;
        const size_t want = blk + static_cast<size_t>(28) * s.K;
        const bool smemp = LDA_FUSE && want + 2048 <= static_cast<size_t>(max_optin);
        s.sweep_smem = smemp ? want : blk;
        s.sweep_fused = smemp;
        const void *fn = nullptr;
        const bool wide = s.K > 16384;  // wide θ entries; p*/P never fit in smem there
        if (wide)
            fn = s.exclude_self ? reinterpret_cast<const void *>(&sweep_kernel<true, false, kTSWide>)
                                : reinterpret_cast<const void *>(&sweep_kernel<false, false, kTSWide>);
        else if (s.exclude_self)
            fn = smemp ? reinterpret_cast<const void *>(&sweep_kernel<true, true>)
                       : reinterpret_cast<const void *>(&sweep_kernel<true, false>);
        else
            fn = smemp ? reinterpret_cast<const void *>(&sweep_kernel<false, true>)
                       : reinterpret_cast<const void *>(&sweep_kernel<false, false>);
        sampler0_fn = fn;  // its attributes are set below only if sampler 0 runs (each first touch of a
                           // kernel loads it: ~ms per kernel on the load path)
    }
    // tile sampler (default): per CTA the n_k histogram, per warp the word
    // table and the batch scratch; <= 8 warps per CTA
    {
        const size_t K4 = static_cast<size_t>((s.K + 3) & ~3);
        s.tile_lmax = std::max(LDA_TILE_LMAX, ((s.K + 1 + 31) / 32 + 3) & ~3);
        const size_t cta = 4 * K4, per_warp = tile_warp_bytes(s.K, s.tile_lmax);
        int wpc = 0;
        while (wpc < LDA_TILE_WPC && cta + per_warp * (wpc + 1) + 1024 <= static_cast<size_t>(max_optin)) ++wpc;
        // sampler -1 (auto): the tile sampler up to K = kTileMaxK; at large K its
        // per-warp tables of 8·K bytes leave too few warps per SM (measured at
        // K = 8192 on the NYTimes shape: sampler 0 is faster)
        if (s.sampler < 0) s.sampler = s.K <= kTileMaxK ? 2 : 3;
        s.sweep_tile = s.sampler == 2 && !s.exclude_self && LDA_FUSE && wpc >= 1 && s.K <= 16384;
        // large K: CTA-shared double-buffered tables (sweep_tile_cta_kernel)
        s.tile_cta_gnk = s.K > kTileMaxK;
        // large K: one CTA per SM with up to 4 compact table buffers, keeping
        // >= 12 warps; else two 8-warp CTAs per SM with 2 buffers each
        const int cmax = s.tile_cta_gnk ? 16 : 8;
        auto fit = [&](int nb) {
            int w = 0;
            while (w < cmax && tile_cta_bytes(s.K, s.tile_lmax, w + 1, s.tile_cta_gnk, nb) + 1024 <=
                                   static_cast<size_t>(max_optin))
                ++w;
            return w;
        };
        s.tile_nbuf = 2;
        if (s.tile_cta_gnk)
            for (int nb = LDA_CTA_NBUF_MAX; nb > 2; --nb)
                if (fit(nb) >= LDA_CTA_MIN_WARPS) {
                    s.tile_nbuf = nb;
                    break;
                }
        const int cwarps = fit(s.tile_nbuf);
        const size_t cta_bytes = tile_cta_bytes(s.K, s.tile_lmax, cwarps, s.tile_cta_gnk, s.tile_nbuf);
        // the tile samplers read θ entries as topic << 18 | count (K <= 16384)
        s.sweep_tile_cta = s.sampler == 3 && !s.exclude_self && LDA_FUSE && cwarps >= 2 && s.K <= 16384;
        if (s.sampler == 3 && !s.sweep_tile_cta) s.sampler = 0;
        if (s.sweep_tile_cta) {
            const void *fn = s.tile_cta_gnk ? reinterpret_cast<const void *>(&sweep_tile_cta_kernel<LDA_TRING_GNK, true>)
                                            : reinterpret_cast<const void *>(&sweep_tile_cta_kernel<LDA_TRING, false>);
            s.tile_block = 32 * cwarps;
            s.tile_smem = cta_bytes;
            if ((e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                          static_cast<int>(s.tile_smem))) != cudaSuccess)
                return e;
            int bps = 1;
            if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, fn, s.tile_block, s.tile_smem)) !=
                cudaSuccess)
                return e;
            s.tile_grid = s.num_sms * (bps > 0 ? bps : 1);
            s.sweep_fused = s.tile_fused;
        }
        s.wt_bytes = s.sweep_tile_cta && s.tile_cta_gnk ? tab_bytes_compact(s.K) : tab_bytes(s.K);
        if (s.sweep_tile || s.sweep_tile_cta) {
            // the variant launch_sweep will use
            const bool compact = s.sweep_tile_cta && s.tile_cta_gnk, vec = (s.K & 3) == 0;
            const void *f = compact ? (vec ? reinterpret_cast<const void *>(&word_table_kernel<true, true>)
                                           : reinterpret_cast<const void *>(&word_table_kernel<false, true>))
                                    : (vec ? reinterpret_cast<const void *>(&word_table_kernel<true, false>)
                                           : reinterpret_cast<const void *>(&word_table_kernel<false, false>));
            if ((e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, 8 * s.K)) != cudaSuccess)
                return e;
        }
        if (s.sweep_tile) {
            const void *fn = reinterpret_cast<const void *>(&sweep_tile_kernel<LDA_TRING>);
            s.tile_block = 32 * wpc;
            s.tile_smem = cta + per_warp * wpc;
            if ((e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                          static_cast<int>(s.tile_smem))) != cudaSuccess)
                return e;
            int bps = 1;
            if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, fn, s.tile_block, s.tile_smem)) !=
                cudaSuccess)
                return e;
            s.tile_grid = s.num_sms * (bps > 0 ? bps : 1);
            s.sweep_fused = s.tile_fused;
        }
    }
    if (!s.sweep_tile && !s.sweep_tile_cta) {
        // sampler 0 runs
        if ((e = cudaFuncSetAttribute(sampler0_fn, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                      static_cast<int>(s.sweep_smem))) != cudaSuccess)
            return e;
        int bps = 1;
        if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, sampler0_fn, kSweepThreads, s.sweep_smem)) !=
            cudaSuccess)
            return e;
        s.sweep_grid = s.num_sms * (bps > 0 ? bps : 1);
    }
    // recount: two K-length histograms per CTA in shared memory, or (wide K)
    // in a global scratch slice per CTA
    s.recount_gmem = static_cast<size_t>(8) * s.K + 1024 > static_cast<size_t>(max_optin);
    if (!s.recount_gmem &&
        (e = cudaFuncSetAttribute(reinterpret_cast<const void *>(&recount_kernel<false>),
                                  cudaFuncAttributeMaxDynamicSharedMemorySize, 8 * s.K)) != cudaSuccess)
        return e;
    // theta: as many warps per block (<= 8) as fit; wide K: per-warp global scratch
    size_t per_warp = static_cast<size_t>(4) * (s.K + (s.K + 31) / 32);
    int wpb = static_cast<int>(std::min<size_t>(8, (static_cast<size_t>(max_optin) - 1024) / per_warp));
    s.theta_gmem = wpb < 1;
    if (s.theta_gmem) {
        s.theta_block = 256;
        s.theta_smem = 0;
        s.theta_grid = s.num_sms * 4;
    } else {
        s.theta_block = 32 * wpb;
        s.theta_smem = per_warp * wpb;
        const void *tf = s.K > 16384 ? reinterpret_cast<const void *>(&theta_kernel<false, kTSWide>)
                                     : reinterpret_cast<const void *>(&theta_kernel<false, kTS>);
        if ((e = cudaFuncSetAttribute(tf, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                      static_cast<int>(s.theta_smem))) != cudaSuccess)
            return e;
        int tb = 1;
        if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&tb, tf, s.theta_block, s.theta_smem)) != cudaSuccess)
            return e;
        s.theta_grid = s.num_sms * (tb > 0 ? tb : 1);
    }
    s.ll_blocks = 2 * s.num_sms;
    return cudaSuccess;
}

int launch_init(const DevState &s, void *stream) {
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    if (!s.tok_crank) {  // tile samplers' layout
        const int g = static_cast<int>(std::min<int64_t>(s.n_titems > 0 ? s.n_titems : 1, 65535));
        init_tile_kernel<<<g, 256, 0, st>>>(s.titems, s.n_titems, s.cbase, s.tok_z, static_cast<uint32_t>(s.K),
                                            static_cast<uint32_t>(s.seed), static_cast<uint32_t>(s.seed >> 32));
        return cudaGetLastError();
    }
    const int grid = static_cast<int>(std::min<int64_t>(s.n_chunks > 0 ? s.n_chunks : 1, 65535));
    init_kernel<<<grid, 256, 0, st>>>(s.chunks, s.n_chunks, s.segs, s.tok_crank, s.tok_z, static_cast<uint32_t>(s.K),
                                      static_cast<uint32_t>(s.seed), static_cast<uint32_t>(s.seed >> 32));
    return cudaGetLastError();
}

// Recount work items [rc0, rc1) (rc1 < 0: all).  `first`: the launch that
// opens the sweep's recount (n_k and the rows of split words zeroed).  The
// word-range pipeline (f1) calls it once per word range, each followed by
// the exchange of that range's rows.
int launch_recount(const DevState &s, void *stream, int *launches, int64_t rc0, int64_t rc1, bool first) {
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    cudaError_t e;
    if (rc1 < 0) rc1 = s.n_rchunks;
    int32_t *nk = s.nwk + static_cast<size_t>(s.V) * s.K;
    if (first) {
        if ((e = cudaMemsetAsync(nk, 0, sizeof(int32_t) * s.K, st)) != cudaSuccess) return e;
        if (s.n_split > 0) {
            zero_rows_kernel<<<static_cast<int>(std::min<int64_t>(s.n_split, 65535)), 256, 0, st>>>(
                s.split_words, s.n_split, s.nwk, s.K);
            ++*launches;
        }
    }
    if (rc1 <= rc0) return cudaGetLastError();
    if ((e = cudaMemsetAsync(s.counter + 1, 0, sizeof(uint32_t), st)) != cudaSuccess) return e;
    const int grid = static_cast<int>(std::min<int64_t>(rc1 - rc0, static_cast<int64_t>(s.num_sms) * s.recount_bps));
    if (s.recount_gmem)
        recount_kernel<true><<<grid, 256, 0, st>>>(s.rchunks + rc0, rc1 - rc0, s.segs, s.K, s.tok_z, s.nwk, nk,
                                                  s.counter + 1, s.recount_scratch);
    else
        recount_kernel<false><<<grid, 256, 8 * s.K, st>>>(s.rchunks + rc0, rc1 - rc0, s.segs, s.K, s.tok_z, s.nwk,
                                                          nk, s.counter + 1, nullptr);
    ++*launches;
    return cudaGetLastError();
}

int launch_tok_row(const DevState &s, void *stream) {
    if (s.D > 0)
        tok_row_kernel<<<static_cast<unsigned>((s.D + 7) / 8), 256, 0, static_cast<cudaStream_t>(stream)>>>(
            s.doc_ptr32, s.row_off32, s.doc_map, s.tok_row, s.D);
    return cudaGetLastError();
}

int launch_gather_z(const DevState &s, uint16_t *zd, void *stream) {
    const int64_t thr = (s.T + 7) / 8;
    if (thr > 0)
        gather_z_kernel<<<static_cast<unsigned>((thr + 255) / 256), 256, 0, static_cast<cudaStream_t>(stream)>>>(
            s.doc_map, s.tok_z, zd, s.T);
    return cudaGetLastError();
}

int launch_scatter_z(const DevState &s, const uint16_t *zd, void *stream) {
    if (s.T > 0)
        scatter_z_kernel<<<4 * s.num_sms, 256, 0, static_cast<cudaStream_t>(stream)>>>(s.doc_map, zd, s.tok_z, s.T);
    return cudaGetLastError();
}

int launch_theta(const DevState &s, unsigned long long *stat_out, void *stream, int *launches) {
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    cudaError_t e;
    if ((e = cudaMemsetAsync(stat_out, 0, 2 * sizeof(unsigned long long), st)) != cudaSuccess) return e;
    const int64_t thr = (s.T + 7) / 8;
    if (thr > 0) {
        gather_z_kernel<<<static_cast<unsigned>((thr + 255) / 256), 256, 0, st>>>(s.doc_map, s.tok_z, s.z_doc, s.T);
        ++*launches;
    }
    if (s.theta_gmem)
        theta_kernel<true, kTSWide><<<s.theta_grid, s.theta_block, 0, st>>>(s.doc_ptr32, s.row_off32, s.z_doc, s.rows,
                                                                           s.D, s.K, stat_out, s.theta_scratch);
    else if (s.K > 16384)
        theta_kernel<false, kTSWide><<<s.theta_grid, s.theta_block, s.theta_smem, st>>>(
            s.doc_ptr32, s.row_off32, s.z_doc, s.rows, s.D, s.K, stat_out, nullptr);
    else
        theta_kernel<false, kTS><<<s.theta_grid, s.theta_block, s.theta_smem, st>>>(
            s.doc_ptr32, s.row_off32, s.z_doc, s.rows, s.D, s.K, stat_out, nullptr);
    ++*launches;
    return cudaGetLastError();
}

int launch_sweep(const DevState &s, uint32_t t, void *stream, int *launches, void *table_done_event, int parts) {
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    cudaError_t e;
    const double Vbeta = static_cast<double>(s.V) * s.beta;
    const int32_t *nk = s.nwk + static_cast<size_t>(s.V) * s.K;
    if (parts & 1) {
        prologue_kernel<<<(s.K + 255) / 256, 256, 0, st>>>(nk, s.K, Vbeta, s.denom);
        ++*launches;
    }
    if (!s.sweep_tile && !s.sweep_tile_cta && table_done_event &&
        (e = cudaEventRecord(static_cast<cudaEvent_t>(table_done_event), st)) != cudaSuccess)
        return e;
    if ((e = cudaMemsetAsync(s.counter, 0, sizeof(uint32_t), st)) != cudaSuccess) return e;
    SweepArgs a;
    if (s.sweep_fused) {
        // next n_wk: rows of words split over chunks (or without tokens) and n_k start at 0
        a.nwk_next = s.nwk_alt;
        a.nk_next = s.nwk_alt + static_cast<size_t>(s.V) * s.K;
        if ((e = cudaMemsetAsync(a.nk_next, 0, sizeof(int32_t) * s.K, st)) != cudaSuccess) return e;
        if (s.n_zero_words > 0) {
            zero_rows_kernel<<<static_cast<int>(std::min<int64_t>(s.n_zero_words, 65535)), 256, 0, st>>>(
                s.zero_words, s.n_zero_words, s.nwk_alt, s.K);
            ++*launches;
        }
    } else {
        a.nwk_next = nullptr;
        a.nk_next = nullptr;
    }
    if (s.sweep_tile || s.sweep_tile_cta) {
        // every row of the next n_wk is accumulated (words span tiles)
        if ((parts & 1) && s.tile_fused &&
            (e = cudaMemsetAsync(s.nwk_alt, 0, sizeof(int32_t) * (static_cast<size_t>(s.V) * s.K + s.K), st)) !=
                cudaSuccess)
            return e;
        const int wtb = static_cast<int>(std::min<int64_t>((static_cast<int64_t>(s.V) + 7) / 8, 8 * s.num_sms));
        const bool compact = s.sweep_tile_cta && s.tile_cta_gnk;
        SparseRows sp{compact ? s.sp_off : nullptr, s.sp_nnz, s.sp_ent, s.s32};
        if (!(parts & 1)) {
            // the tables of this sweep are built (out-of-HBM chunks after the first)
        } else if ((s.K & 3) == 0 && compact)
            word_table_kernel<true, true><<<wtb, 256, 8 * s.K, st>>>(s.nwk, s.denom, s.V, s.K, s.alpha, s.beta,
                                                                     s.wtab, sp);
        else if (compact)
            word_table_kernel<false, true><<<wtb, 256, 8 * s.K, st>>>(s.nwk, s.denom, s.V, s.K, s.alpha, s.beta,
                                                                      s.wtab, sp);
        else if ((s.K & 3) == 0)
            word_table_kernel<true, false><<<wtb, 256, 8 * s.K, st>>>(s.nwk, s.denom, s.V, s.K, s.alpha, s.beta,
                                                                      s.wtab, sp);
        else
            word_table_kernel<false, false><<<wtb, 256, 8 * s.K, st>>>(s.nwk, s.denom, s.V, s.K, s.alpha, s.beta,
                                                                       s.wtab, sp);
        if (parts & 1) ++*launches;
        if (table_done_event && (e = cudaEventRecord(static_cast<cudaEvent_t>(table_done_event), st)) != cudaSuccess)
            return e;
        if (!(parts & 2)) return cudaGetLastError();
        TileArgs ta;
        ta.items = s.titems;
        ta.n_items = s.n_titems;
        ta.cbase = s.cbase;
        ta.tok_row = s.tok_row;
        ta.z = s.tok_z;
        ta.rows = s.rows;
        ta.nwk = s.nwk;
        ta.denom = s.denom;
        ta.counter = s.counter;
        ta.nwk_next = s.nwk_alt;
        ta.nk_next = s.nwk_alt + static_cast<size_t>(s.V) * s.K;
        ta.n_exact = s.stat + 2;
        ta.K = s.K;
        ta.alpha = s.alpha;
        ta.beta = s.beta;
        ta.lmax = s.tile_lmax;
        ta.slack = s.certify_slack;
        ta.wtab = s.wtab;
        ta.wt_bytes = static_cast<uint32_t>(s.wt_bytes);
        ta.nbuf = s.tile_nbuf;
        ta.recount = s.tile_fused ? 1 : 0;
        ta.sp_off = sp.off;
        ta.sp_nnz = s.sp_nnz;
        ta.sp_ent = s.sp_ent;
        ta.s32 = s.s32;
        ta.t = t;
        uint32_t k0 = static_cast<uint32_t>(s.seed), k1 = static_cast<uint32_t>(s.seed >> 32);
        for (int r = 0; r < 10; ++r) {
            ta.key0[r] = k0;
            ta.key1[r] = k1;
            k0 += 0x9E3779B9u;
            k1 += 0xBB67AE85u;
        }
        if (s.sweep_tile_cta && s.tile_cta_gnk)
            sweep_tile_cta_kernel<LDA_TRING_GNK, true><<<s.tile_grid, s.tile_block, s.tile_smem, st>>>(ta);
        else if (s.sweep_tile_cta)
            sweep_tile_cta_kernel<LDA_TRING, false><<<s.tile_grid, s.tile_block, s.tile_smem, st>>>(ta);
        else
            sweep_tile_kernel<LDA_TRING><<<s.tile_grid, s.tile_block, s.tile_smem, st>>>(ta);
        ++*launches;
        return cudaGetLastError();
    }
    a.chunks = s.chunks;
    a.n_chunks = s.n_chunks;
    a.segs = s.segs;
    a.tok_row = s.tok_row;
    a.tok_crank = s.tok_crank;
    a.z = s.tok_z;
    a.rows = reinterpret_cast<const uint4 *>(s.rows);
    a.nwk = s.nwk;
    a.nk = nk;
    a.denom = s.denom;
    a.counter = s.counter;
    a.gscratch = s.sweep_fused ? nullptr : s.sweep_scratch;
    a.K = s.K;
    a.alpha = s.alpha;
    a.beta = s.beta;
    a.Vbeta = Vbeta;
    a.t = t;
    uint32_t k0 = static_cast<uint32_t>(s.seed), k1 = static_cast<uint32_t>(s.seed >> 32);
    for (int r = 0; r < 10; ++r) {
        a.key0[r] = k0;
        a.key1[r] = k1;
        k0 += 0x9E3779B9u;
        k1 += 0xBB67AE85u;
    }
    if (s.K > 16384) {
        if (s.exclude_self) sweep_kernel<true, false, kTSWide><<<s.sweep_grid, kSweepThreads, s.sweep_smem, st>>>(a);
        else sweep_kernel<false, false, kTSWide><<<s.sweep_grid, kSweepThreads, s.sweep_smem, st>>>(a);
    } else if (s.exclude_self) {
        if (s.sweep_fused) sweep_kernel<true, true><<<s.sweep_grid, kSweepThreads, s.sweep_smem, st>>>(a);
        else sweep_kernel<true, false><<<s.sweep_grid, kSweepThreads, s.sweep_smem, st>>>(a);
    } else {
        if (s.sweep_fused) sweep_kernel<false, true><<<s.sweep_grid, kSweepThreads, s.sweep_smem, st>>>(a);
        else sweep_kernel<false, false><<<s.sweep_grid, kSweepThreads, s.sweep_smem, st>>>(a);
    }
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
    ll_doc_kernel<<<s.ll_blocks, 256, 0, st>>>(s.doc_ptr32, s.row_off32, s.rows, s.D, s.alpha, lgamma(s.alpha),
                                               Kalpha, lgamma(Kalpha), pd);
    ++*launches;
    ll_final_kernel<<<1, 256, 0, st>>>(pw, nw, pd, s.ll_blocks, s.nwk + static_cast<size_t>(s.V) * s.K, s.K,
                                       Vbeta, lgamma(Vbeta), word_part ? 1 : 0, s.ll_out);
    ++*launches;
    return cudaGetLastError();
}

}  // namespace lda
