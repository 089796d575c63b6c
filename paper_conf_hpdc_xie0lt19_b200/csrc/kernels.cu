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

#include <cstdint>

#include "lda_internal.h"

namespace lda {

constexpr unsigned kFull = 0xffffffffu;
constexpr int kSweepThreads = 256;
constexpr int kMaxBlk = 16;  // block-end prefixes kept per token for the sparse rescan
#ifndef LDA_RING
#define LDA_RING 6
#endif
#ifndef LDA_SWEEP_MINB
#define LDA_SWEEP_MINB 3
#endif
constexpr int kRing = LDA_RING;  // 16-byte row quads in flight per sampler lane

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

// Bring [p, p + bytes) into L2 without a register or scoreboard slot (one
// bulk-prefetch instruction per θ row; bytes a multiple of 16).
__device__ __forceinline__ void prefetch_l2_bulk(const void *p, uint32_t bytes) {
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(p), "r"(bytes) : "memory");
}

// Word-major position of virtual index v of a word, walking the word's runs
// forward from run s (v must not decrease between calls with the same s).
__device__ __forceinline__ uint32_t run_position(const Seg *__restrict__ segs, uint32_t &s, uint32_t v) {
    while (segs[s + 1].vstart <= v) ++s;
    return segs[s].pos + (v - segs[s].vstart);
}

// ---------------------------------------------------------------------------
// a1: random initial assignment (L377-379; X10): z = (x0·K) >> 32, t = 0.
// ---------------------------------------------------------------------------
__global__ void init_kernel(const SampleChunk *__restrict__ chunks, int64_t n_chunks,
                            const Seg *__restrict__ segs, uint16_t *__restrict__ z, uint32_t K, uint32_t k0,
                            uint32_t k1) {
    for (int64_t ci = blockIdx.x; ci < n_chunks; ci += gridDim.x) {
        const SampleChunk ch = chunks[ci];
        uint32_t sg = ch.seg0;
        for (uint32_t j = threadIdx.x; j < ch.count; j += blockDim.x) {
            const uint32_t x0 = philox_x0(ch.c_base + j, 0u, k0, k1);
            z[run_position(segs, sg, ch.vbegin + j)] =
                static_cast<uint16_t>((static_cast<uint64_t>(x0) * K) >> 32);
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
// θ rows: word 0 = nnz, words 1..nnz = topic << 16 | count (ascending topics,
// X7), zero words up to the next 32-byte boundary.
// ---------------------------------------------------------------------------
struct SweepArgs {
    const SampleChunk *chunks;
    int64_t n_chunks;
    const Seg *segs;
    const uint32_t *tok_row;
    uint16_t *z;
    const uint4 *rows;
    const int32_t *nwk;
    const int32_t *nk;
    const double *denom;
    uint32_t *counter;
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

template <bool EXCL>
struct Mass {
    // mass of one θ entry e = topic << 16 | count under the word's p*
    __device__ __forceinline__ static double fma_into(uint32_t e, const double *__restrict__ pstar, int zo,
                                                      double po_new, double acc) {
        const uint32_t tp = e >> 16;
        uint32_t cn = e & 0xFFFFu;
        double p = pstar[tp];
        if (EXCL && static_cast<int>(tp) == zo && cn != 0u) {
            cn -= 1u;
            p = po_new;
        }
        return fma(static_cast<double>(cn), p, acc);
    }
};

template <bool EXCL>
__global__ void __launch_bounds__(kSweepThreads, LDA_SWEEP_MINB) sweep_kernel(SweepArgs a) {
    extern __shared__ double smem_d[];
    __shared__ int s_ci;
    __shared__ double s_wtot[kSweepThreads / 32];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int K = a.K;
    // smem: [blkC: kMaxBlk x 256 fp64][p*: K][P: K] (p*/P in global scratch for large K)
    double *blkC = smem_d;
    double *pstar = a.gscratch ? a.gscratch + static_cast<size_t>(blockIdx.x) * 2 * K
                               : smem_d + kMaxBlk * kSweepThreads;
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
        // row is streamed in 16-byte quads through a ring of kRing quads held
        // in registers, so ~kRing·16 B per thread are in flight (a 32-byte
        // block = 2 quads; words past nnz in the last block are zero).
        uint32_t sg = ch.seg0;
        for (uint32_t j = tid; j < ch.count; j += kSweepThreads) {
            const uint32_t p = run_position(a.segs, sg, ch.vbegin + j);
            const uint32_t row = __ldg(a.tok_row + p);
            const uint4 *r = a.rows + static_cast<size_t>(row) * 2;
            uint4 q[kRing];
            q[0] = ld_nc_v4(r);            // header quad: nnz + 3 entries
#pragma unroll
            for (int i = 1; i < kRing; ++i) q[i] = make_uint4(0u, 0u, 0u, 0u);
            q[1] = ld_nc_v4(r + 1);        // every row has >= 1 block = 2 quads
            const uint32_t x0 = philox_x0_sched(ch.c_base + j, a.t, a.key0, a.key1);
            int zo = 0;
            double po_new = 0.0, delta = 0.0;
            if (EXCL) {
                zo = static_cast<int>(a.z[p]);
                po_new = (static_cast<double>(nwk_row[zo] - 1) + a.beta) /
                         (static_cast<double>(a.nk[zo] - 1) + a.Vbeta);
                delta = a.alpha * po_new - a.alpha * pstar[zo];
            }
            const uint32_t len = q[0].x;
            const uint32_t nblk = (len + 8u) >> 3;   // 32-byte blocks holding words 0..len
            const uint32_t nq = 2u * nblk;           // quads to stream (zero-padded tail)
#pragma unroll
            for (int i = 2; i < kRing; ++i)
                if (static_cast<uint32_t>(i) < nq) q[i] = ld_nc_v4(r + i);
            // pass 1: S over the row, block-end prefixes to smem
            double S = 0.0;
            S = Mass<EXCL>::fma_into(q[0].y, pstar, zo, po_new, S);
            S = Mass<EXCL>::fma_into(q[0].z, pstar, zo, po_new, S);
            S = Mass<EXCL>::fma_into(q[0].w, pstar, zo, po_new, S);
            q[0] = (static_cast<uint32_t>(kRing) < nq) ? ld_nc_v4(r + kRing) : make_uint4(0u, 0u, 0u, 0u);
            // quads 1 .. nq-1, ring slot (qi % kRing); qi odd ends a block
            for (uint32_t base = 0; base < nq; base += kRing) {
#pragma unroll
                for (int i = 0; i < kRing; ++i) {
                    const uint32_t qi = base + i;
                    if (qi == 0) continue;
                    if (qi >= nq) break;
                    const uint4 u = q[i];
                    const uint32_t nx = qi + kRing;
                    q[i] = (nx < nq) ? ld_nc_v4(r + nx) : make_uint4(0u, 0u, 0u, 0u);
                    S = Mass<EXCL>::fma_into(u.x, pstar, zo, po_new, S);
                    S = Mass<EXCL>::fma_into(u.y, pstar, zo, po_new, S);
                    S = Mass<EXCL>::fma_into(u.z, pstar, zo, po_new, S);
                    S = Mass<EXCL>::fma_into(u.w, pstar, zo, po_new, S);
                    if (qi & 1u) {
                        const uint32_t b = qi >> 1;
                        if (b < kMaxBlk) blkC[b * kSweepThreads + tid] = S;
                    }
                }
            }
            const double U = static_cast<double>(x0) * 2.3283064365386962890625e-10;  // x0 · 2^-32
            const double x = U * (S + (EXCL ? Q + delta : Q));
            int z;
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
        C = Mass<EXCL>::fma_into((e), pstar, zo, po_new, C);          \
        if (z < 0 && C > x) z = static_cast<int>((e) >> 16);          \
    }
                for (; z < 0 && b < nblk; ++b) {  // one block, or a linear tail past kMaxBlk
                    const uint4 u0 = ld_nc_v4(r + 2 * b), u1 = ld_nc_v4(r + 2 * b + 1);
                    if (b > 0) LDA_STEP(u0.x)
                    LDA_STEP(u0.y) LDA_STEP(u0.z) LDA_STEP(u0.w)
                    LDA_STEP(u1.x) LDA_STEP(u1.y) LDA_STEP(u1.z) LDA_STEP(u1.w)
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
        }
        __syncthreads();
    }
}

// ---------------------------------------------------------------------------
// a3 + a4, TMA-staged variant (the default sampler).
//
// Same arithmetic as sweep_kernel, but the θ rows are moved by the Tensor
// Memory Accelerator instead of per-thread loads: each warp draws 32 tokens
// at a time (one sampler per lane); a lane first loads its row's 32-byte
// header block (nnz + 7 entries), then issues ONE cp.async.bulk copy of the
// rest of its row into the warp's shared-memory stage, completing on an
// mbarrier.  Two stages per warp: the bulk copies of batch i+1 and the header
// loads of batch i+2 are in flight while batch i is drawn from shared memory,
// so the memory system sees ~2 x 32 whole rows in flight per warp with no
// registers tied up (the direct-load sampler above keeps ~1 block per thread
// in flight and is latency-bound).
// ---------------------------------------------------------------------------
constexpr int kTW = 4;                // warps per CTA
constexpr int kTThreads = 32 * kTW;   // 128
constexpr int kTCap = 288;            // staged 32-byte blocks per warp per stage (~9 per lane)

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
__device__ __forceinline__ void tma_row_to_smem(void *dst, const void *src, uint32_t bytes, uint64_t *bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
            smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar))
        : "memory");
}

struct TBatch {
    uint32_t p;     // word-major position of the lane's token
    uint32_t row;   // θ row of its document, 32-byte units
    uint4 h0, h1;   // row block 0: nnz + 7 entries
    uint32_t off;   // first staged block in the warp's stage
    uint32_t nst;   // staged blocks (row blocks 1..nst)
    bool valid;
};

template <bool EXCL>
__global__ void __launch_bounds__(kTThreads) sweep_tma_kernel(SweepArgs a) {
    extern __shared__ __align__(128) unsigned char smem_t[];
    __shared__ uint64_t mbar[2][kTW];
    __shared__ int s_ci;
    __shared__ double s_wtot[kTW];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int K = a.K;
    // smem: [stage 0: kTW x kTCap x 32 B][stage 1][blkC: kMaxBlk x 128 fp64][p*: K][P: K]
    uint4 *stage0 = reinterpret_cast<uint4 *>(smem_t);
    double *blkC = reinterpret_cast<double *>(smem_t + 2 * kTW * kTCap * 32);
    double *pstar = a.gscratch ? a.gscratch + static_cast<size_t>(blockIdx.x) * 2 * K : blkC + kMaxBlk * kTThreads;
    double *P = pstar + K;
    const int E = (K + kTThreads - 1) / kTThreads;
    if (lane == 0) {
        mbar_init(&mbar[0][warp], 1);
        mbar_init(&mbar[1][warp], 1);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    __syncthreads();
    uint32_t parity[2] = {0u, 0u};
    int cur_word = -1;

    for (;;) {
        if (tid == 0) s_ci = static_cast<int>(atomicAdd(a.counter, 1u));
        __syncthreads();
        const int ci = s_ci;
        if (ci >= a.n_chunks) break;
        const SampleChunk ch = a.chunks[ci];
        const int32_t *nwk_row = a.nwk + static_cast<size_t>(ch.word) * K;

        if (static_cast<int>(ch.word) != cur_word) {
            // p*(k) = (n_wk + β)/(n_k + Vβ) and the inclusive prefix of α·p*(k) (Eq. 8)
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

        // this warp's batches: tokens j = (i*kTW + warp)*32 + lane
        uint32_t sg = ch.seg0;
        auto load_header = [&](uint32_t i, TBatch &B) {
            const uint32_t j = (i * kTW + warp) * 32u + lane;
            B.valid = j < ch.count;
            B.h0 = make_uint4(0u, 0u, 0u, 0u);
            B.h1 = B.h0;
            if (B.valid) {
                B.p = run_position(a.segs, sg, ch.vbegin + j);
                B.row = __ldg(a.tok_row + B.p);
                const uint4 *r = a.rows + static_cast<size_t>(B.row) * 2;
                B.h0 = ld_nc_v4(r);
                B.h1 = ld_nc_v4(r + 1);
            }
        };
        auto issue_body = [&](int s, TBatch &B) {
            const uint32_t nblk = B.valid ? ((B.h0.x + 8u) >> 3) : 0u;
            const uint32_t need = nblk ? nblk - 1u : 0u;
            uint32_t incl = need;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t y = __shfl_up_sync(kFull, incl, o);
                if (lane >= o) incl += y;
            }
            const uint32_t total = __shfl_sync(kFull, incl, 31);
            B.off = incl - need;
            B.nst = B.off >= static_cast<uint32_t>(kTCap) ? 0u : min(need, kTCap - B.off);
            const uint32_t staged = min(total, static_cast<uint32_t>(kTCap));
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            __syncwarp();
            if (lane == 0) mbar_arrive_expect_tx(&mbar[s][warp], staged * 32u);
            __syncwarp();
            if (B.nst) {
                uint4 *dst = stage0 + (static_cast<size_t>(s) * kTW + warp) * kTCap * 2 + B.off * 2;
                tma_row_to_smem(dst, a.rows + static_cast<size_t>(B.row) * 2 + 2, B.nst * 32u, &mbar[s][warp]);
            }
        };

        const uint32_t nb = ch.count > static_cast<uint32_t>(warp) * 32u
                                ? (ch.count - warp * 32u + kTW * 32u - 1u) / (kTW * 32u)
                                : 0u;
        TBatch Bc, Bn, Bnn;
        if (nb > 0) {
            load_header(0, Bc);
            issue_body(0, Bc);
            if (nb > 1) load_header(1, Bn);
        }
        for (uint32_t i = 0; i < nb; ++i) {
            const int s = static_cast<int>(i & 1u);
            if (i + 1 < nb) issue_body(s ^ 1, Bn);
            if (i + 2 < nb) load_header(i + 2, Bnn);
            mbar_wait(&mbar[s][warp], parity[s]);
            parity[s] ^= 1u;

            if (Bc.valid) {
                const uint4 *stg = stage0 + (static_cast<size_t>(s) * kTW + warp) * kTCap * 2 + Bc.off * 2;
                const uint4 *gr = a.rows + static_cast<size_t>(Bc.row) * 2;
                const uint32_t j = (i * kTW + warp) * 32u + lane;
                const uint32_t x0 = philox_x0_sched(ch.c_base + j, a.t, a.key0, a.key1);
                int zo = 0;
                double po_new = 0.0, delta = 0.0;
                if (EXCL) {
                    zo = static_cast<int>(a.z[Bc.p]);
                    po_new = (static_cast<double>(nwk_row[zo] - 1) + a.beta) /
                             (static_cast<double>(a.nk[zo] - 1) + a.Vbeta);
                    delta = a.alpha * po_new - a.alpha * pstar[zo];
                }
                const uint32_t len = Bc.h0.x;
                const uint32_t nblk = (len + 8u) >> 3;
                // block b >= 1 of the row: staged copy, or global memory past the stage
#define LDA_BLOCK(b, u0, u1)                                                     \
    if ((b) <= Bc.nst) {                                                         \
        u0 = stg[2 * ((b) - 1)];                                                 \
        u1 = stg[2 * ((b) - 1) + 1];                                             \
    } else {                                                                     \
        u0 = ld_nc_v4(gr + 2 * (b));                                             \
        u1 = ld_nc_v4(gr + 2 * (b) + 1);                                         \
    }
                double S = 0.0;
                S = Mass<EXCL>::fma_into(Bc.h0.y, pstar, zo, po_new, S);
                S = Mass<EXCL>::fma_into(Bc.h0.z, pstar, zo, po_new, S);
                S = Mass<EXCL>::fma_into(Bc.h0.w, pstar, zo, po_new, S);
                S = Mass<EXCL>::fma_into(Bc.h1.x, pstar, zo, po_new, S);
                S = Mass<EXCL>::fma_into(Bc.h1.y, pstar, zo, po_new, S);
                S = Mass<EXCL>::fma_into(Bc.h1.z, pstar, zo, po_new, S);
                S = Mass<EXCL>::fma_into(Bc.h1.w, pstar, zo, po_new, S);
                blkC[tid] = S;
                for (uint32_t b = 1; b < nblk; ++b) {
                    uint4 u0, u1;
                    LDA_BLOCK(b, u0, u1)
                    S = Mass<EXCL>::fma_into(u0.x, pstar, zo, po_new, S);
                    S = Mass<EXCL>::fma_into(u0.y, pstar, zo, po_new, S);
                    S = Mass<EXCL>::fma_into(u0.z, pstar, zo, po_new, S);
                    S = Mass<EXCL>::fma_into(u0.w, pstar, zo, po_new, S);
                    S = Mass<EXCL>::fma_into(u1.x, pstar, zo, po_new, S);
                    S = Mass<EXCL>::fma_into(u1.y, pstar, zo, po_new, S);
                    S = Mass<EXCL>::fma_into(u1.z, pstar, zo, po_new, S);
                    S = Mass<EXCL>::fma_into(u1.w, pstar, zo, po_new, S);
                    if (b < kMaxBlk) blkC[b * kTThreads + tid] = S;
                }
                const double U = static_cast<double>(x0) * 2.3283064365386962890625e-10;  // x0 · 2^-32
                const double x = U * (S + (EXCL ? Q + delta : Q));
                int z;
                if (x < S) {
                    const uint32_t nbk = nblk < kMaxBlk ? nblk : kMaxBlk;
                    uint32_t b = 0;
                    while (b < nbk && !(blkC[b * kTThreads + tid] > x)) ++b;
                    double C = b == 0 ? 0.0 : blkC[(b - 1) * kTThreads + tid];
                    z = -1;
#define LDA_STEP(e)                                                   \
    {                                                                 \
        C = Mass<EXCL>::fma_into((e), pstar, zo, po_new, C);          \
        if (z < 0 && C > x) z = static_cast<int>((e) >> 16);          \
    }
                    if (b == 0) {
                        LDA_STEP(Bc.h0.y) LDA_STEP(Bc.h0.z) LDA_STEP(Bc.h0.w)
                        LDA_STEP(Bc.h1.x) LDA_STEP(Bc.h1.y) LDA_STEP(Bc.h1.z) LDA_STEP(Bc.h1.w)
                        b = 1;
                    }
                    for (; z < 0 && b < nblk; ++b) {
                        uint4 u0, u1;
                        LDA_BLOCK(b, u0, u1)
                        LDA_STEP(u0.x) LDA_STEP(u0.y) LDA_STEP(u0.z) LDA_STEP(u0.w)
                        LDA_STEP(u1.x) LDA_STEP(u1.y) LDA_STEP(u1.z) LDA_STEP(u1.w)
                    }
#undef LDA_STEP
                    if (z < 0) z = K - 1;  // unreachable: the last entry's prefix is S > x
                } else {
                    int lo = 0, hi = K - 1;
                    while (lo < hi) {
                        const int mid = (lo + hi) >> 1;
                        double pk = P[mid];
                        if (EXCL && mid >= zo) pk += delta;
                        if (S + pk > x) hi = mid;
                        else lo = mid + 1;
                    }
                    z = lo;
                }
#undef LDA_BLOCK
                a.z[Bc.p] = static_cast<uint16_t>(z);
            }
            __syncwarp();
            Bc = Bn;
            Bn = Bnn;
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
                               const Seg *__restrict__ segs, int K, const uint16_t *__restrict__ z,
                               int32_t *__restrict__ nwk, int32_t *__restrict__ nk,
                               uint32_t *__restrict__ counter) {
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
        const uint32_t w = c.word & 0x7FFFFFFFu;
        const bool split = (c.word >> 31) != 0u;
        uint32_t sg = c.seg0;
        for (uint32_t j = threadIdx.x; j < c.vcount; j += blockDim.x)
            atomicAdd(&hist[z[run_position(segs, sg, c.vbegin + j)]], 1);
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
        if (nkp[k]) atomicAdd(nk + k, nkp[k]);
}

// ---------------------------------------------------------------------------
// a5: θ rebuild.  One warp per document: gather z through the doc-word map,
// count topics in a per-warp shared histogram + bitmap, then write the row
// as ascending (topic << 16 | count) entries with a popc scan over the bitmap.
// O(L_d + K/32) per document instead of the paper's dense O(K) row.
// ---------------------------------------------------------------------------
// Two-phase variant, phase A: z in document order, zd[i] = z[doc_map[i]]
// (independent gathers with high memory-level parallelism, in doc order).
__global__ void gather_z_kernel(const uint32_t *__restrict__ doc_map, const uint16_t *__restrict__ z,
                                uint16_t *__restrict__ zd, int64_t T) {
    const int64_t i0 = (static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x) * 4;
    if (i0 + 3 < T) {
        const uint4 m = __ldcs(reinterpret_cast<const uint4 *>(doc_map + i0));
        const uint16_t a = z[m.x], b = z[m.y], c = z[m.z], d = z[m.w];
        ushort4 o;
        o.x = a; o.y = b; o.z = c; o.w = d;
        *reinterpret_cast<ushort4 *>(zd + i0) = o;
    } else {
        for (int64_t i = i0; i < T; ++i) zd[i] = z[doc_map[i]];
    }
}

// GATHERED = false: z through the doc-word map (fused); true: zd is z in
// document order (phase B of the two-phase variant).
template <bool GATHERED>
__global__ void theta_kernel(const uint32_t *__restrict__ doc_ptr32, const uint32_t *__restrict__ row_off32,
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
            const uint32_t k = GATHERED ? z[i] : z[doc_map[i]];
            atomicAdd(&cnt[k], 1u);
            atomicOr(&bits[k >> 5], 1u << (k & 31));
        }
        __syncwarp();
        uint32_t *row = rows + static_cast<size_t>(row_off32[d]) * 8;
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
        // zero the words after the last entry up to the 32-byte boundary
        const uint32_t pad = (8u - ((1u + base) & 7u)) & 7u;
        if (static_cast<uint32_t>(lane) < pad) row[1 + base + lane] = 0u;
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
// Launchers
// ---------------------------------------------------------------------------
int configure_kernels(DevState &s) {
    cudaError_t e;
    int dev = 0;
    if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
    if ((e = cudaDeviceGetAttribute(&s.num_sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess) return e;
    int max_optin = 0;
    if ((e = cudaDeviceGetAttribute(&max_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev)) != cudaSuccess)
        return e;
    // sampler
    if (s.sampler == 1) {
        const size_t fixed = 2 * kTW * kTCap * 32 + sizeof(double) * kMaxBlk * kTThreads;
        const size_t want = fixed + static_cast<size_t>(16) * s.K;
        s.sweep_smem = (want + 2048 <= static_cast<size_t>(max_optin)) ? want : fixed;
        s.sweep_block = kTThreads;
        const void *fns[2] = {reinterpret_cast<const void *>(&sweep_tma_kernel<false>),
                              reinterpret_cast<const void *>(&sweep_tma_kernel<true>)};
        for (int i = 0; i < 2; ++i)
            if ((e = cudaFuncSetAttribute(fns[i], cudaFuncAttributeMaxDynamicSharedMemorySize,
                                          static_cast<int>(s.sweep_smem))) != cudaSuccess)
                return e;
        int bps = 1;
        if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, fns[s.exclude_self ? 1 : 0], kTThreads,
                                                               s.sweep_smem)) != cudaSuccess)
            return e;
        s.sweep_grid = s.num_sms * (bps > 0 ? bps : 1);
    } else {
        const size_t blk = sizeof(double) * kMaxBlk * kSweepThreads;
        size_t want = blk + static_cast<size_t>(16) * s.K;
        s.sweep_smem = (want + 2048 <= static_cast<size_t>(max_optin)) ? want : blk;
        s.sweep_block = kSweepThreads;
        const void *fns[2] = {reinterpret_cast<const void *>(&sweep_kernel<false>),
                              reinterpret_cast<const void *>(&sweep_kernel<true>)};
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
    }
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
    if ((e = cudaFuncSetAttribute(reinterpret_cast<const void *>(&theta_kernel<true>),
                                  cudaFuncAttributeMaxDynamicSharedMemorySize,
                                  static_cast<int>(s.theta_smem))) != cudaSuccess)
        return e;
    if ((e = cudaFuncSetAttribute(reinterpret_cast<const void *>(&theta_kernel<false>),
                                  cudaFuncAttributeMaxDynamicSharedMemorySize,
                                  static_cast<int>(s.theta_smem))) != cudaSuccess)
        return e;
    int tb = 1;
    if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&tb, reinterpret_cast<const void *>(&theta_kernel<false>),
                                                           s.theta_block, s.theta_smem)) != cudaSuccess)
        return e;
    s.theta_grid = s.num_sms * (tb > 0 ? tb : 1);
    s.ll_blocks = 2 * s.num_sms;
    return cudaSuccess;
}

int launch_init(const DevState &s, void *stream) {
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    const int grid = static_cast<int>(std::min<int64_t>(s.n_chunks > 0 ? s.n_chunks : 1, 65535));
    init_kernel<<<grid, 256, 0, st>>>(s.chunks, s.n_chunks, s.segs, s.tok_z, static_cast<uint32_t>(s.K),
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
        s.rchunks, s.n_rchunks, s.segs, s.K, s.tok_z, s.nwk, nk, s.counter + 1);
    ++*launches;
    return cudaGetLastError();
}

int launch_theta(const DevState &s, unsigned long long *stat_out, void *stream, int *launches) {
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    cudaError_t e;
    if ((e = cudaMemsetAsync(stat_out, 0, 2 * sizeof(unsigned long long), st)) != cudaSuccess) return e;
    if (s.z_doc) {
        const int64_t thr = (s.T + 3) / 4;
        gather_z_kernel<<<static_cast<unsigned>((thr + 255) / 256), 256, 0, st>>>(s.doc_map, s.tok_z, s.z_doc, s.T);
        ++*launches;
        theta_kernel<true><<<s.theta_grid, s.theta_block, s.theta_smem, st>>>(s.doc_ptr32, s.row_off32, s.doc_map,
                                                                           s.z_doc, s.rows, s.D, s.K, stat_out);
    } else {
        theta_kernel<false><<<s.theta_grid, s.theta_block, s.theta_smem, st>>>(s.doc_ptr32, s.row_off32, s.doc_map,
                                                                            s.tok_z, s.rows, s.D, s.K, stat_out);
    }
    ++*launches;
    return cudaGetLastError();
}

int launch_sweep(const DevState &s, uint32_t t, void *stream, int *launches) {
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    cudaError_t e;
    const double Vbeta = static_cast<double>(s.V) * s.beta;
    const int32_t *nk = s.nwk + static_cast<size_t>(s.V) * s.K;
    prologue_kernel<<<(s.K + 255) / 256, 256, 0, st>>>(nk, s.K, Vbeta, s.denom);
    ++*launches;
    if ((e = cudaMemsetAsync(s.counter, 0, sizeof(uint32_t), st)) != cudaSuccess) return e;
    SweepArgs a;
    a.chunks = s.chunks;
    a.n_chunks = s.n_chunks;
    a.segs = s.segs;
    a.tok_row = s.tok_row;
    a.z = s.tok_z;
    a.rows = reinterpret_cast<const uint4 *>(s.rows);
    a.nwk = s.nwk;
    a.nk = nk;
    a.denom = s.denom;
    a.counter = s.counter;
    a.gscratch = s.sweep_scratch;  // non-null only when p*/P do not fit in smem
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
    if (s.sampler == 1) {
        if (s.exclude_self)
            sweep_tma_kernel<true><<<s.sweep_grid, kTThreads, s.sweep_smem, st>>>(a);
        else
            sweep_tma_kernel<false><<<s.sweep_grid, kTThreads, s.sweep_smem, st>>>(a);
    } else {
        if (s.exclude_self)
            sweep_kernel<true><<<s.sweep_grid, kSweepThreads, s.sweep_smem, st>>>(a);
        else
            sweep_kernel<false><<<s.sweep_grid, kSweepThreads, s.sweep_smem, st>>>(a);
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
