"""Byte models shared by bench.py, the tools and the tests.  The bench runs
the library's defaults (no lda_set_option calls): the timed configuration is
the one lda_create -> lda_load_corpus -> lda_iterate gives every user."""

# Algorithmic bytes per sweep, per GPU:
#   B_alg = T_g·20 + 4·Σ_t nnz_{d(t)} + 8·V·K + 4·Σ_d nnz'_d + 8·D_g
# and the part of it the sampling kernel moves (dominant kernel):
#   B_sample = T_g·(4 doc id + 8 row bounds + 2 z_new) + 4·Σ_t nnz_{d(t)} + 4·V·K
def bytes_sweep(T, D, V, K, sum_nnz_tok, sum_nnz_doc_new):
    return 20 * T + 4 * sum_nnz_tok + 8 * V * K + 4 * sum_nnz_doc_new + 8 * D


def bytes_sample(T, V, K, sum_nnz_tok):
    return 14 * T + 4 * sum_nnz_tok + 4 * V * K
