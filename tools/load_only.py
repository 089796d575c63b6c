"""Load a BASELINE config through lda_load_corpus twice (no sweeps) and print
the load times; for profiling the load path (a0) under ncu.
    python tools/load_only.py --config pubmed"""
import argparse
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_hpdc_xie0lt19_b200 as L  # noqa: E402
from paper_conf_hpdc_xie0lt19_b200 import synth  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="pubmed")
ap.add_argument("--reps", type=int, default=2)
ap.add_argument("--pinned", action="store_true", help="words and doc_ptr in page-locked memory (as bench.py)")
args = ap.parse_args()
cfg = synth.CONFIGS[args.config]
torch.cuda.set_device(0)
dp, w, _ = synth.generate_config(cfg, "cuda")
doc_ptr = dp.cpu().numpy().astype(np.int64)
words = w.cpu().numpy().astype(np.int32)
del dp, w
torch.cuda.empty_cache()
if args.pinned:
    pw = torch.empty(len(words), dtype=torch.int32, pin_memory=True)
    pw.numpy()[:] = words
    words = pw.numpy()
for r in range(args.reps):
    t0 = time.time()
    m = L.LDA(cfg.D, cfg.V, cfg.K, cfg.alpha, cfg.beta, device=0)
    m.load(doc_ptr, words, cfg.seed)
    print(f"load {r}: {time.time() - t0:.3f} s", flush=True)
    m.close()
