"""Experiment driver (GPU box): generate one synthetic corpus, then time the
sampler under several lda_set_option sets in one process.

    python tools/exp_options.py --config pubmed --sweeps 5 --warmup 3 \
        --set "fused_recount=0" --set "fused_recount=1"

Prints one line per option set: G tokens/s, ms per phase, nnz per token.
Not a bench number (no clocks check, no e2e); bench.py is the contract.
"""
import argparse
import json
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_hpdc_xie0lt19_b200 as L  # noqa: E402
from paper_conf_hpdc_xie0lt19_b200 import config as C  # noqa: E402
from paper_conf_hpdc_xie0lt19_b200 import synth  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="pubmed")
    ap.add_argument("--sweeps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--set", action="append", default=[])
    args = ap.parse_args()
    cfg = synth.CONFIGS[args.config]
    torch.cuda.set_device(0)
    t0 = time.time()
    dp, w, _ = synth.generate_config(cfg, "cuda")
    doc_ptr = dp.cpu().numpy().astype(np.int64)
    words = w.cpu().numpy().astype(np.int32)
    del dp, w
    torch.cuda.empty_cache()
    print(f"# {cfg.name}: generated in {time.time() - t0:.1f}s, lib {L.LIB_PATH}", flush=True)
    sets = args.set or [""]
    for s in sets:
        opts = {}
        for kv in filter(None, s.split(",")):
            k, v = kv.split("=")
            opts[k] = int(v)
        t1 = time.time()
        m = L.LDA(cfg.D, cfg.V, cfg.K, cfg.alpha, cfg.beta, device=0, **opts)
        m.load(doc_ptr, words, cfg.seed)
        tl = time.time() - t1
        m.iterate(args.warmup)
        m.iterate(args.sweeps)
        st = m.stats()
        log = m.sweep_log()
        n = args.sweeps
        ms = st["ms_total"] / n
        nnz = float(np.mean(log["sum_nnz_tok"])) / cfg.T
        bs = np.mean([C.bytes_sample(cfg.T, cfg.V, cfg.K, int(x)) for x in log["sum_nnz_tok"]])
        out = {"set": s, "Gtok_s": round(cfg.T / ms / 1e6, 3), "ms": round(ms, 3),
               "sample": round(st["ms_sample"] / n, 3), "table": round(st["ms_table"] / n, 3), "theta": round(st["ms_theta"] / n, 3),
               "recount": round(st["ms_recount"] / n, 3), "nnz": round(nnz, 2),
               "sample_GBs": round(bs / (st["ms_sample"] / n / 1e3) / 1e9, 1), "load_s": round(tl, 1),
               "n_exact_per_sweep": st["n_exact_redraws"] / n, "ll": round(m.loglik(), 5)}
        print(json.dumps(out), flush=True)
        m.close()


if __name__ == "__main__":
    main()
