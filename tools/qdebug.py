"""Debug: fallback counters of the quad sampler (variants/qdbg.so)."""
import ctypes, os, sys
import numpy as np
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ["LDA_LIBRARY"] = os.path.join(ROOT, "variants", "qdbg.so")
import paper_conf_hpdc_xie0lt19_b200 as L
from paper_conf_hpdc_xie0lt19_b200 import synth
cfg = synth.scaled(synth.CONFIGS["pubmed"], 0.02)
dp, w = synth.to_numpy(*synth.generate_config(cfg, "cuda"))[:2]
m = L.LDA(cfg.D, cfg.V, cfg.K, cfg.alpha, cfg.beta, device=0)
m.load(dp, w, cfg.seed)
for it in range(4):
    m.iterate(1)
    c = (ctypes.c_ulonglong * 8)()
    L.lib().lda_debug_counters(c)
    print(it, "n_exact", m.stats()["n_exact_redraws"], "T", cfg.T, "counters", list(c), flush=True)
