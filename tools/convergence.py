#!/usr/bin/env python
"""Convergence vs. time: per-token log-likelihood of the
model against cumulative sampling time, the analogue of the paper's Fig. 8
(LL vs. time) for our own system on the synthetic shapes
(there are no comparison systems or real corpora here).

    python tools/convergence.py --config pubmed --sweeps 100 --every 5
    python -m torch.distributed.run --nproc-per-node N --master-addr 127.0.0.1 \
        tools/convergence.py --config pubmed ...

Every `every` sweeps: cumulative device time of the sweeps (CUDA events on the
library stream, max over ranks), LL/token (reading X11: the collapsed joint,
Griffiths-Steyvers), Σnnz/T, and the sweeps' tokens/s.  LL evaluation is not
timed (as in the paper's figure).  Prints one JSON line per point and writes
profiles/convergence_<config>_<N>gpu.md when --write is given.

--anchor (small corpora; a config may be downscaled as name@fraction, e.g.
nytimes@0.01): the CPU oracle (oracle-omp, bit-identical to the
single-threaded oracle) runs the same chain and its LL/token is reported
beside the GPU's at every point (test infrastructure: the oracle is only
called here as the anchor of the curve, never on the product path).
"""
import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def _config(name):
    from paper_conf_hpdc_xie0lt19_b200 import synth
    if "@" in name:
        base, frac = name.split("@")
        return synth.scaled(synth.CONFIGS[base], float(frac), name)
    return synth.CONFIGS[name]


def run(config="tiny", sweeps=20, every=5, device_index=None, write=False, opts=None, quiet=False,
        anchor=False):
    import torch
    import torch.distributed as dist

    import paper_conf_hpdc_xie0lt19_b200 as L
    from paper_conf_hpdc_xie0lt19_b200 import synth

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0")) if device_index is None else device_index
    torch.cuda.set_device(local)
    if world > 1 and not dist.is_initialized():
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    cfg = _config(config)
    dp_t, w_t, _ = synth.generate_config(cfg, torch.device("cuda", local) if cfg.T > 10_000_000 else "cpu")
    doc_ptr_full = dp_t.cpu().numpy().astype(np.int64)
    words_full = w_t.cpu().numpy().astype(np.int32)
    del dp_t, w_t
    bounds = L.lda_partition_docs(doc_ptr_full, world)
    d0, d1 = int(bounds[rank]), int(bounds[rank + 1])
    t0, t1 = int(doc_ptr_full[d0]), int(doc_ptr_full[d1])
    o = {}
    o.update(opts or {})
    m = L.LDA(cfg.D, cfg.V, cfg.K, cfg.alpha, cfg.beta, device=local, **o)
    if world > 1:
        obj = [L.lda_nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        m.init_dist(rank, world, obj[0])
    m.load((doc_ptr_full[d0:d1 + 1] - t0).astype(np.int64), words_full[t0:t1], cfg.seed, d0, d1)
    orc = None
    if anchor and rank == 0:
        from oracle import oracle as O
        orc = O.OracleLDA(cfg.D, cfg.V, cfg.K, cfg.alpha, cfg.beta).load(doc_ptr_full, words_full, cfg.seed)
    pts = []
    t_cum = 0.0
    ll = m.loglik()
    pts.append({"sweep": 0, "ms": 0.0, "ll_per_token": ll, "nnz_per_token": None, "tokens_per_s": None,
                "oracle_ll": orc.loglik() if orc else None})
    done = 0
    while done < sweeps:
        n = min(every, sweeps - done)
        m.iterate(n)
        done += n
        st = m.stats()
        log = m.sweep_log()
        ms = torch.tensor([st["ms_total"]], dtype=torch.float64, device=torch.device("cuda", local))
        if world > 1:
            dist.all_reduce(ms, op=dist.ReduceOp.MAX)
        t_cum += float(ms.item())
        ll = m.loglik()
        if orc is not None:
            orc.iterate(n, parallel=True)
        pt = {"sweep": done, "ms": round(t_cum, 3), "ll_per_token": ll,
              "nnz_per_token": float(np.mean(log["sum_nnz_tok"])) / max(t1 - t0, 1),
              "tokens_per_s": cfg.T * n / (float(ms.item()) / 1e3),
              "oracle_ll": orc.loglik() if orc is not None else None}
        pts.append(pt)
        if rank == 0 and not quiet:
            print(json.dumps({"config": cfg.name, "n_gpus": world, **pt}), flush=True)
    m.close()
    if rank == 0 and write:
        os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
        path = os.path.join(ROOT, "profiles", f"convergence_{cfg.name.replace('@', '_')}_{world}gpu.md")
        with open(path, "w") as f:
            f.write(f"# LL/token vs. sampling time — {cfg.name}, K={cfg.K}, {world} GPU(s)\n\n")
            f.write("`tools/convergence.py` (Fig. 8 analogue; device time of the sweeps only, LL untimed).\n\n")
            if anchor:
                f.write("Oracle anchor: the CPU oracle (oracle-omp) runs the same chain; its LL/token beside "
                        "the GPU's.\n\n")
            f.write("| sweep | cumulative ms | LL/token | oracle LL/token | nnz/token | tokens/s (last interval) |\n"
                    "|---|---|---|---|---|---|\n")
            for p in pts:
                nnz = "" if p["nnz_per_token"] is None else f"{p['nnz_per_token']:.2f}"
                tps = "" if p["tokens_per_s"] is None else f"{p['tokens_per_s'] / 1e9:.3f} G"
                ol = "" if p.get("oracle_ll") is None else f"{p['oracle_ll']:.8f}"
                f.write(f"| {p['sweep']} | {p['ms']:.1f} | {p['ll_per_token']:.8f} | {ol} | {nnz} | {tps} |\n")
    if world > 1 and dist.is_initialized():
        dist.destroy_process_group()
    return pts


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="pubmed")
    ap.add_argument("--sweeps", type=int, default=100)
    ap.add_argument("--every", type=int, default=5)
    ap.add_argument("--write", action="store_true")
    ap.add_argument("--opt", action="append", default=[])
    ap.add_argument("--anchor", action="store_true", help="run the CPU oracle beside (small corpora)")
    a = ap.parse_args()
    opts = {k: int(v) for k, v in (kv.split("=") for kv in a.opt)}
    t = time.time()
    run(a.config, a.sweeps, a.every, write=a.write, opts=opts, anchor=a.anchor)
    if int(os.environ.get("RANK", "0")) == 0:
        print(f"# wall {time.time() - t:.1f} s", flush=True)


if __name__ == "__main__":
    main()
