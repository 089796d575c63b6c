"""Diagnostics (variants/liblda_stats.so, built with LDA_TILE_STATS=1): the
tile sampler's batches per sweep -- tokens, θ-row lines walked, distinct rows,
walk steps -- on a bench config.  Usage (GPU box):
    LDA_LIBRARY=variants/liblda_stats.so python tools/tile_stats.py pubmed 25"""
import ctypes
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_hpdc_xie0lt19_b200 as L  # noqa: E402
from paper_conf_hpdc_xie0lt19_b200 import synth  # noqa: E402

cfg = synth.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "pubmed"]
warm = int(sys.argv[2]) if len(sys.argv) > 2 else 25
dp, w, _ = synth.generate_config(cfg, "cuda")
doc_ptr, words = synth.to_numpy(dp, w)
del dp, w
torch.cuda.empty_cache()
m = L.LDA(cfg.D, cfg.V, cfg.K, cfg.alpha, cfg.beta, device=0).load(doc_ptr, words, cfg.seed)
m.iterate(warm)
f = L.lib().lda_debug_tile_stats
out = (ctypes.c_ulonglong * 8)()
f(out, 1)
m.iterate(1)
f(out, 0)
b, t, l, r, s = out[0], out[1], out[2], out[3], out[4]
st = m.stats()
print(f"{cfg.name} sweep {warm + 1}: batches {b} tokens {t} (T {cfg.T}) tokens/batch {t / b:.2f} "
      f"lines/batch {l / b:.1f} rows/batch {r / b:.1f} lines/row {l / r:.2f} steps/batch {s / b:.2f} "
      f"nnz/token {st['sum_nnz_tok'] / cfg.T:.1f} items {st['n_sample_chunks']}")
