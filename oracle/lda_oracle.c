/*
 * oracle/lda_oracle.c — plain, slow, single-threaded CPU oracle for the
 * CuLDA_CGS hot path: the collapsed Gibbs sampling (CGS) sweep of LDA.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.
 * It shares no code, header, table or constant generator with the CUDA
 * product path (paper_conf_hpdc_xie0lt19_b200/csrc); neither includes the
 * other.
 *
 * Source of truth: /root/reference/PAPER.md (cited "L<n>", the paged
 * transcript line) and the readings of SURVEY.md §8(c) (cited "X<n>"), which
 * DESIGN.md lists.  Arithmetic is IEEE fp64, no FMA contraction
 * (-ffp-contract=off), sequential sums in the order the paper's equations
 * write them.
 *
 * Notation (paper -> here): θ_{d,k} -> n_dk, ϕ_{k,v} -> n_wk (w = v),
 * Σ_v ϕ_{k,v} -> n_k, DocLen_d -> L_d.  Tokens are addressed two ways:
 *   input order   i : doc-major, i = doc_ptr[d] + j            (the corpus)
 *   canonical     c : position in the stable sort by (w, d, j)  (X18, §8(c)2;
 *                     the paper's "word-first order", L1189-1191)
 *
 * Pin status (what each function is checked against in tests/):
 *   orc_philox4x32_10 ... Random123 known-answer vectors (Salmon et al. SC'11)
 *   orc_search ........... Fig. 5 worked example (L1065-1107) + edge cases
 *   orc_draw / sweeps .... one-sweep chi^2 vs Eq. 1 closed form; exact
 *                          posterior chi^2 (SEQUENTIAL); exact stationary law
 *                          of the synchronous chain (SWEEP); SURVEY App. A
 *                          golden vectors (independent implementation)
 *   orc_counts ........... Eq. 5 (L1011-1015) and the row/column-sum
 *                          invariants; brute-force recount
 *   orc_loglik ........... K=1 Dirichlet-multinomial closed form; scipy
 *                          gammaln brute force; topic-relabelling invariance
 * No function is "parity unpinned".
 */
#include <math.h>
#ifdef _OPENMP
#include <omp.h>
#endif
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* ------------------------------------------------------------------------ */
/* Philox4x32-10 (Salmon, Moraes, Dror, Shaw, SC'11).  The paper does not   */
/* name its RNG (X9); both sides implement this counter-based generator.     */
/* ------------------------------------------------------------------------ */

void orc_philox4x32_10(const uint32_t ctr_in[4], const uint32_t key_in[2],
                       uint32_t out[4])
{
    uint32_t c0 = ctr_in[0], c1 = ctr_in[1], c2 = ctr_in[2], c3 = ctr_in[3];
    uint32_t k0 = key_in[0], k1 = key_in[1];
    for (int round = 0; round < 10; round++) {
        uint64_t prod0 = (uint64_t)0xD2511F53u * (uint64_t)c0;
        uint64_t prod1 = (uint64_t)0xCD9E8D57u * (uint64_t)c2;
        uint32_t hi0 = (uint32_t)(prod0 >> 32), lo0 = (uint32_t)prod0;
        uint32_t hi1 = (uint32_t)(prod1 >> 32), lo1 = (uint32_t)prod1;
        uint32_t n0 = hi1 ^ c1 ^ k0;
        uint32_t n1 = lo1;
        uint32_t n2 = hi0 ^ c3 ^ k1;
        uint32_t n3 = lo0;
        c0 = n0; c1 = n1; c2 = n2; c3 = n3;
        k0 += 0x9E3779B9u;   /* Weyl key schedule */
        k1 += 0xBB67AE85u;
    }
    out[0] = c0; out[1] = c1; out[2] = c2; out[3] = c3;
}

/* The one random word a token uses at sweep t (X9): key = (seed lo, seed hi),
 * counter = (c lo, c hi, t, 0), output word x0.  t = 0 is the random
 * initialisation (L377-379), t = 1, 2, ... are the sweeps. */
uint32_t orc_token_x0(uint64_t seed, uint64_t c, uint32_t t)
{
    uint32_t ctr[4] = {(uint32_t)c, (uint32_t)(c >> 32), t, 0u};
    uint32_t key[2] = {(uint32_t)seed, (uint32_t)(seed >> 32)};
    uint32_t out[4];
    orc_philox4x32_10(ctr, key, out);
    return out[0];
}

/* ------------------------------------------------------------------------ */
/* Corpus order                                                              */
/* ------------------------------------------------------------------------ */

/* Canonical index of every input token: a stable sort of the doc-major
 * corpus by word id, i.e. order (w, d, j) (L1189-1191 "sort the tokens in a
 * word-first order"; tie order X18).  canon[i] for input token i. */
void orc_canonical_order(int64_t D, int32_t V, const int64_t *doc_ptr,
                         const int32_t *words, int64_t *canon)
{
    int64_t T = doc_ptr[D];
    int64_t *next = (int64_t *)calloc((size_t)V + 1, sizeof(int64_t));
    for (int64_t i = 0; i < T; i++) next[words[i] + 1] += 1;
    for (int32_t w = 0; w < V; w++) next[w + 1] += next[w];   /* start of w */
    for (int64_t i = 0; i < T; i++) canon[i] = next[words[i]]++;
    free(next);
}

/* Canonical index of selected input tokens only (for sampled checks at
 * full size): one scan over the corpus, same definition as above. */
void orc_canonical_index_of(int64_t D, int32_t V, const int64_t *doc_ptr,
                            const int32_t *words, int64_t n_query,
                            const int64_t *query_sorted /* ascending */,
                            int64_t *canon_out)
{
    int64_t T = doc_ptr[D];
    int64_t *start = (int64_t *)calloc((size_t)V + 1, sizeof(int64_t));
    int64_t *seen = (int64_t *)calloc((size_t)V, sizeof(int64_t));
    for (int64_t i = 0; i < T; i++) start[words[i] + 1] += 1;
    for (int32_t w = 0; w < V; w++) start[w + 1] += start[w];
    int64_t q = 0;
    for (int64_t i = 0; i < T && q < n_query; i++) {
        int32_t w = words[i];
        while (q < n_query && query_sorted[q] == i) {
            canon_out[q] = start[w] + seen[w];
            q++;
        }
        seen[w] += 1;
    }
    free(start);
    free(seen);
}

/* ------------------------------------------------------------------------ */
/* Random initial assignment (L377-379; X10): z = floor(U * K) computed      */
/* exactly as (x0 * K) >> 32.                                                */
/* ------------------------------------------------------------------------ */

uint16_t orc_init_topic(uint64_t seed, uint64_t c, int32_t K)
{
    uint32_t x0 = orc_token_x0(seed, c, 0u);
    return (uint16_t)(((uint64_t)x0 * (uint64_t)K) >> 32);
}

void orc_init(int64_t T, const int64_t *canon, int32_t K, uint64_t seed,
              uint16_t *z /* input order */)
{
    for (int64_t i = 0; i < T; i++) z[i] = orc_init_topic(seed, (uint64_t)canon[i], K);
}

/* z of every token of one word, in canonical order: word w's tokens occupy
 * canonical positions [c_begin, c_begin + n).  Used to build n_wk at init at
 * full size without sorting. */
void orc_init_range_hist(uint64_t seed, int64_t c_begin, int64_t n, int32_t K,
                         int32_t *hist /* K, accumulated */)
{
    for (int64_t c = c_begin; c < c_begin + n; c++)
        hist[orc_init_topic(seed, (uint64_t)c, K)] += 1;
}

/* ------------------------------------------------------------------------ */
/* Counts: θ (n_dk, dense D x K here), ϕ (n_wk, V x K row-major by word,     */
/* X13) and n_k, rebuilt from z (§6.2 "model update", L1271-1309).           */
/* ------------------------------------------------------------------------ */

void orc_counts(int64_t D, int32_t V, int32_t K, const int64_t *doc_ptr,
                const int32_t *words, const uint16_t *z, int32_t *n_wk,
                int32_t *n_k, int32_t *n_dk /* D*K or NULL */)
{
    memset(n_wk, 0, sizeof(int32_t) * (size_t)V * (size_t)K);
    memset(n_k, 0, sizeof(int32_t) * (size_t)K);
    if (n_dk) memset(n_dk, 0, sizeof(int32_t) * (size_t)D * (size_t)K);
    for (int64_t d = 0; d < D; d++) {
        for (int64_t i = doc_ptr[d]; i < doc_ptr[d + 1]; i++) {
            int32_t w = words[i], k = z[i];
            n_wk[(int64_t)w * K + k] += 1;
            n_k[k] += 1;
            if (n_dk) n_dk[d * K + k] += 1;
        }
    }
}

/* Returns 0 if every invariant holds: Eq. 5 (Σ_k n_dk = L_d, L1011-1015),
 * Σ_k n_wk = #tokens of w, n_k = Σ_w n_wk, all counts >= 0. */
int orc_check_invariants(int64_t D, int32_t V, int32_t K, const int64_t *doc_ptr,
                         const int32_t *words, const int32_t *n_wk,
                         const int32_t *n_k, const int32_t *n_dk)
{
    int64_t T = doc_ptr[D];
    int64_t *wc = (int64_t *)calloc((size_t)V, sizeof(int64_t));
    int64_t *col = (int64_t *)calloc((size_t)K, sizeof(int64_t));
    int bad = 0;
    for (int64_t i = 0; i < T; i++) wc[words[i]] += 1;
    for (int32_t w = 0; w < V && !bad; w++) {
        int64_t s = 0;
        for (int32_t k = 0; k < K; k++) {
            int32_t v = n_wk[(int64_t)w * K + k];
            if (v < 0) bad = 1;
            s += v;
            col[k] += v;
        }
        if (s != wc[w]) bad = 2;
    }
    for (int32_t k = 0; k < K && !bad; k++)
        if (col[k] != n_k[k]) bad = 3;
    if (n_dk) {
        for (int64_t d = 0; d < D && !bad; d++) {
            int64_t s = 0;
            for (int32_t k = 0; k < K; k++) {
                if (n_dk[d * K + k] < 0) bad = 4;
                s += n_dk[d * K + k];
            }
            if (s != doc_ptr[d + 1] - doc_ptr[d]) bad = 5;
        }
    }
    free(wc);
    free(col);
    return bad;
}

/* ------------------------------------------------------------------------ */
/* The draw                                                                  */
/* ------------------------------------------------------------------------ */

/* Tree-based sampling turned into a search (Fig. 5): the first
 * bin whose inclusive prefix exceeds x ("the minimal k that makes
 * prefixSum[k] > u"; strict >, X6).  Returns n if no bin exceeds x. */
int64_t orc_search(const double *prefix, int64_t n, double x)
{
    for (int64_t b = 0; b < n; b++)
        if (prefix[b] > x) return b;
    return n;
}

/* One token's new topic (Eq. 1 L399-409 via the split of Eq. 6-8,
 * L1019-1031 and L1253-1269; Alg. 2; readings X2-X8):
 *   p*(k) = (n'_wk + β) / (n'_k + Vβ)                 (Eq. 8)
 *   bins  = [sparse: n'_dk p*(k) for k ascending with frozen n_dk > 0]  (p1)
 *           ++ [dense: α p*(k) for k = 0..K-1]                          (p2)
 *   C     = inclusive prefix of the bins, sequential; total = C_last
 *           (so S = C at the last sparse bin, S + Q = total; Eq. 7)
 *   x     = U * total with U = x0 * 2^-32              (one uniform, X4/X8)
 *   z     = topic of the first bin with C > x; K-1 if none (rounding; X6)
 * Equivalent to Alg. 2's branch "u < S/(S+Q)" then a draw inside the chosen
 * bucket (X5).  n' = n except with exclude_self, where the token's own
 * z_old is removed from all three counts (X2; optional variant).
 * *margin_out = min over bins |x - C_bin| / total (distance of the uniform
 * to the nearest CDF boundary, for the excused-mismatch rule). */
int32_t orc_draw(int32_t K, int32_t V, double alpha, double beta,
                 const int32_t *nwk_row, const int32_t *n_k,
                 const int32_t *ndk_row /* dense K, frozen */,
                 int exclude_self, int32_t z_old, uint32_t x0,
                 double *margin_out)
{
    double Vbeta = (double)V * beta;
    /* pass 1: total (sequential, bins in order) */
    double C = 0.0;
    for (int32_t k = 0; k < K; k++) {
        if (ndk_row[k] > 0) {
            int32_t own = (exclude_self && k == z_old) ? 1 : 0;
            double pstar = ((double)(nwk_row[k] - own) + beta) /
                           ((double)(n_k[k] - own) + Vbeta);
            C = C + (double)(ndk_row[k] - own) * pstar;
        }
    }
    for (int32_t k = 0; k < K; k++) {
        int32_t own = (exclude_self && k == z_old) ? 1 : 0;
        double pstar = ((double)(nwk_row[k] - own) + beta) /
                       ((double)(n_k[k] - own) + Vbeta);
        C = C + alpha * pstar;
    }
    double total = C;
    double U = (double)x0 * (1.0 / 4294967296.0);
    double x = U * total;
    /* pass 2: recompute the identical prefix, pick the first C > x */
    int32_t z = -1;
    double margin = INFINITY;
    C = 0.0;
    for (int32_t k = 0; k < K; k++) {
        if (ndk_row[k] > 0) {
            int32_t own = (exclude_self && k == z_old) ? 1 : 0;
            double pstar = ((double)(nwk_row[k] - own) + beta) /
                           ((double)(n_k[k] - own) + Vbeta);
            C = C + (double)(ndk_row[k] - own) * pstar;
            if (z < 0 && C > x) z = k;
            double m = fabs(x - C) / total;
            if (m < margin) margin = m;
        }
    }
    for (int32_t k = 0; k < K; k++) {
        int32_t own = (exclude_self && k == z_old) ? 1 : 0;
        double pstar = ((double)(nwk_row[k] - own) + beta) /
                       ((double)(n_k[k] - own) + Vbeta);
        C = C + alpha * pstar;
        if (z < 0 && C > x) z = k;
        double m = fabs(x - C) / total;
        if (m < margin) margin = m;
    }
    if (z < 0) z = K - 1;
    if (margin_out) *margin_out = margin;
    return z;
}

/* ------------------------------------------------------------------------ */
/* Sweeps                                                                    */
/* ------------------------------------------------------------------------ */

/* SWEEP mode = one iteration as the paper defines it (L415-421: "a full pass
 * of all tokens as a iteration ... After each iteration, the model θ and ϕ
 * are updated"; X3): every token draws against the counts frozen at the
 * start of the sweep, then all counts are rebuilt from the new z.
 * z (input order) and the counts are updated in place; t >= 1 is the global
 * sweep number (Philox counter word 2). */
/* The draws of one sweep for the tokens of documents [d_begin, d_end) only,
 * against the given (frozen, global) counts; z_new receives their new topics
 * (input order, indexed like z).  A partition of the documents across ranks
 * draws exactly what one process draws (the multi-GPU decomposition, Eq. 4
 * L935-937: each rank samples its documents against the same replicated ϕ). */
void orc_draw_docs(int64_t d_begin, int64_t d_end, int32_t V, int32_t K, double alpha,
                   double beta, const int64_t *doc_ptr, const int32_t *words,
                   const int64_t *canon, uint64_t seed, uint32_t t, int exclude_self,
                   const uint16_t *z, const int32_t *n_wk, const int32_t *n_k,
                   const int32_t *n_dk /* dense D*K, global doc index */,
                   uint16_t *z_new, double *margin)
{
    for (int64_t d = d_begin; d < d_end; d++) {
        for (int64_t i = doc_ptr[d]; i < doc_ptr[d + 1]; i++) {
            int32_t w = words[i];
            uint32_t x0 = orc_token_x0(seed, (uint64_t)canon[i], t);
            double m;
            z_new[i] = (uint16_t)orc_draw(K, V, alpha, beta, n_wk + (int64_t)w * K,
                                          n_k, n_dk + d * K, exclude_self, z[i], x0, &m);
            if (margin) margin[i] = m;
        }
    }
}

void orc_sweep(int64_t D, int32_t V, int32_t K, double alpha, double beta,
               const int64_t *doc_ptr, const int32_t *words, const int64_t *canon,
               uint64_t seed, uint32_t t, int exclude_self, uint16_t *z,
               int32_t *n_wk, int32_t *n_k, int32_t *n_dk, double *margin)
{
    int64_t T = doc_ptr[D];
    uint16_t *z_new = (uint16_t *)malloc(sizeof(uint16_t) * (size_t)(T > 0 ? T : 1));
    orc_draw_docs(0, D, V, K, alpha, beta, doc_ptr, words, canon, seed, t, exclude_self, z,
                  n_wk, n_k, n_dk, z_new, margin);
    memcpy(z, z_new, sizeof(uint16_t) * (size_t)T);
    free(z_new);
    orc_counts(D, V, K, doc_ptr, words, z, n_wk, n_k, n_dk);
}

/* oracle-omp (optional): the same SWEEP with the documents'
 * draws spread over the host cores (OpenMP; without -fopenmp the pragma is
 * ignored and this is orc_sweep).  Every draw reads only the counts frozen at
 * the start of the sweep and its own counter-based uniform (X3, X9), so the
 * order of the documents cannot change any result: z and the counts are
 * bit-identical to orc_sweep's (pinned in tests/test_oracle_pins.py).  Used
 * only to make the 100-sweep LL parity run on a 1M-token corpus tractable. */
void orc_sweep_omp(int64_t D, int32_t V, int32_t K, double alpha, double beta,
                   const int64_t *doc_ptr, const int32_t *words, const int64_t *canon,
                   uint64_t seed, uint32_t t, int exclude_self, uint16_t *z,
                   int32_t *n_wk, int32_t *n_k, int32_t *n_dk, double *margin)
{
    int64_t T = doc_ptr[D];
    uint16_t *z_new = (uint16_t *)malloc(sizeof(uint16_t) * (size_t)(T > 0 ? T : 1));
    int64_t d;
#pragma omp parallel for schedule(dynamic, 64)
    for (d = 0; d < D; d++)
        orc_draw_docs(d, d + 1, V, K, alpha, beta, doc_ptr, words, canon, seed, t, exclude_self, z,
                      n_wk, n_k, n_dk, z_new, margin);
    memcpy(z, z_new, sizeof(uint16_t) * (size_t)T);
    free(z_new);
    orc_counts(D, V, K, doc_ptr, words, z, n_wk, n_k, n_dk);
}

/* number of threads orc_sweep_omp uses (1 without OpenMP) */
int orc_omp_threads(void)
{
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

/* SEQUENTIAL mode: textbook collapsed Gibbs sampling (CGS, L389-409 "CGS
 * iteratively picks up one token ... and reassigns a new topic"; [13, 32]):
 * visit tokens in canonical (word-first) order; remove the token from the
 * counts, draw with the same bin rule, add it back at the new topic.
 * Validation only: this is the chain whose stationary law is the exact
 * posterior p(z | w). */
void orc_sweep_sequential(int64_t D, int32_t V, int32_t K, double alpha,
                          double beta, const int64_t *doc_ptr,
                          const int32_t *words, const int64_t *canon,
                          uint64_t seed, uint32_t t, uint16_t *z, int32_t *n_wk,
                          int32_t *n_k, int32_t *n_dk)
{
    int64_t T = doc_ptr[D];
    int64_t *input_of = (int64_t *)malloc(sizeof(int64_t) * (size_t)(T > 0 ? T : 1));
    int64_t *doc_of = (int64_t *)malloc(sizeof(int64_t) * (size_t)(T > 0 ? T : 1));
    for (int64_t d = 0; d < D; d++)
        for (int64_t i = doc_ptr[d]; i < doc_ptr[d + 1]; i++) {
            input_of[canon[i]] = i;
            doc_of[i] = d;
        }
    for (int64_t c = 0; c < T; c++) {
        int64_t i = input_of[c], d = doc_of[i];
        int32_t w = words[i], k = z[i];
        n_wk[(int64_t)w * K + k] -= 1;
        n_k[k] -= 1;
        n_dk[d * K + k] -= 1;
        uint32_t x0 = orc_token_x0(seed, (uint64_t)c, t);
        int32_t kn = orc_draw(K, V, alpha, beta, n_wk + (int64_t)w * K, n_k,
                              n_dk + d * K, 0, -1, x0, NULL);
        z[i] = (uint16_t)kn;
        n_wk[(int64_t)w * K + kn] += 1;
        n_k[kn] += 1;
        n_dk[d * K + kn] += 1;
    }
    free(input_of);
    free(doc_of);
}

/* ------------------------------------------------------------------------ */
/* Log-likelihood (Fig. 8 plots "log-likelihood/token", L1509-1519, without  */
/* a formula; X11): the collapsed joint log p(w, z | α, β) of Griffiths &    */
/* Steyvers, written out term by term:                                       */
/*   K lgΓ(Vβ) − Σ_k lgΓ(n_k + Vβ) + Σ_k Σ_w [lgΓ(n_wk + β) − lgΓ(β)]        */
/* + D lgΓ(Kα) − Σ_d lgΓ(L_d + Kα) + Σ_d Σ_k [lgΓ(n_dk + α) − lgΓ(α)]        */
/* Returned divided by T (per token).                                        */
/* ------------------------------------------------------------------------ */

double orc_loglik(int64_t D, int32_t V, int32_t K, double alpha, double beta,
                  const int64_t *doc_ptr, const int32_t *n_wk, const int32_t *n_k,
                  const int32_t *n_dk)
{
    double Vbeta = (double)V * beta, Kalpha = (double)K * alpha;
    double word_part = (double)K * lgamma(Vbeta);
    for (int32_t k = 0; k < K; k++) word_part -= lgamma((double)n_k[k] + Vbeta);
    for (int32_t w = 0; w < V; w++)
        for (int32_t k = 0; k < K; k++)
            word_part += lgamma((double)n_wk[(int64_t)w * K + k] + beta) - lgamma(beta);
    double doc_part = (double)D * lgamma(Kalpha);
    for (int64_t d = 0; d < D; d++) {
        doc_part -= lgamma((double)(doc_ptr[d + 1] - doc_ptr[d]) + Kalpha);
        for (int32_t k = 0; k < K; k++)
            doc_part += lgamma((double)n_dk[d * K + k] + alpha) - lgamma(alpha);
    }
    int64_t T = doc_ptr[D];
    return (word_part + doc_part) / (double)(T > 0 ? T : 1);
}

/* ------------------------------------------------------------------------ */
/* Many independent chains on a tiny corpus (statistical pins only).         */
/* Chain r uses seed = seed0 + r.  If z_start is NULL each chain starts from */
/* its own random init (t = 0); otherwise from z_start.  mode 0 = SWEEP,     */
/* 1 = SEQUENTIAL.  Final states go to z_final[r*T + i] (input order).       */
/* ------------------------------------------------------------------------ */

void orc_run_chains(int64_t D, int32_t V, int32_t K, double alpha, double beta,
                    const int64_t *doc_ptr, const int32_t *words,
                    const int64_t *canon, uint64_t seed0, int64_t n_chains,
                    int32_t n_sweeps, int mode, int exclude_self,
                    const uint16_t *z_start, uint16_t *z_final)
{
    int64_t T = doc_ptr[D];
    int32_t *n_wk = (int32_t *)malloc(sizeof(int32_t) * (size_t)V * K);
    int32_t *n_k = (int32_t *)malloc(sizeof(int32_t) * (size_t)K);
    int32_t *n_dk = (int32_t *)malloc(sizeof(int32_t) * (size_t)D * K);
    for (int64_t r = 0; r < n_chains; r++) {
        uint64_t seed = seed0 + (uint64_t)r;
        uint16_t *z = z_final + r * T;
        if (z_start) memcpy(z, z_start, sizeof(uint16_t) * (size_t)T);
        else orc_init(T, canon, K, seed, z);
        orc_counts(D, V, K, doc_ptr, words, z, n_wk, n_k, n_dk);
        for (int32_t s = 1; s <= n_sweeps; s++) {
            if (mode == 0)
                orc_sweep(D, V, K, alpha, beta, doc_ptr, words, canon, seed,
                          (uint32_t)s, exclude_self, z, n_wk, n_k, n_dk, NULL);
            else
                orc_sweep_sequential(D, V, K, alpha, beta, doc_ptr, words, canon,
                                     seed, (uint32_t)s, z, n_wk, n_k, n_dk);
        }
    }
    free(n_wk);
    free(n_k);
    free(n_dk);
}
