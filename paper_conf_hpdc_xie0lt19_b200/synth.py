"""Seeded synthetic corpora with the shapes of the paper's workloads.

This module holds NONE of the sampler's arithmetic: it only draws corpora
from LDA's generative process with a Zipf word base (SURVEY.md §8(d)
"Synthetic inputs"), so the CUDA path and the oracle can be fed the same
arrays.  Shapes follow Table 3: NYTimes T=99,542,125,
D=299,752, V=101,636; PubMed T=737,869,083, D=8,200,000, V=141,043.

Recipe:
  * word base        pi_v ∝ (v+1)^-s, s = 1
  * topic-word       phi_k ~ Dirichlet(eta_scale · V · pi),   k < K_gen
  * doc-topic        theta_d ~ Dirichlet(alpha_gen = 0.1)
  * doc lengths      L_d = round(LogNormal(ln(T/D) − σ²/2, σ)) clamped to
                     [1, 65535], then ±1 on random docs until Σ L_d = T
  * tokens           z ~ theta_d, w ~ phi_z by inverse CDF
All draws come from one torch.Generator seeded with ``corpus_seed`` on the
requested device (CPU for the small parity configs, CUDA for the full-size
bench configs; the two devices' streams differ, the shapes do not).
"""
from __future__ import annotations

import math
from dataclasses import dataclass

import numpy as np
import torch


@dataclass(frozen=True)
class CorpusConfig:
    name: str
    D: int
    V: int
    T: int
    sigma: float
    K: int
    K_gen: int
    corpus_seed: int
    seed: int = 1           # sampler seed (Philox key)
    sweeps: int = 20

    @property
    def alpha(self) -> float:      # α = 50/K (reading X1)
        return 50.0 / self.K

    @property
    def beta(self) -> float:       # β = 0.01 (L413-415, L1339)
        return 0.01


# BASELINE.json "configs" (index in brackets) and SURVEY.md §8(d) table.
CONFIGS = {
    # [0] tiny: the oracle finishes all 20 sweeps in seconds
    "tiny": CorpusConfig("tiny", 1000, 500, 50_000, 0.5, 16, 16, 1, 1, 20),
    # [1] NYTimes-shaped, K = 1024
    "nytimes": CorpusConfig("nytimes", 299_752, 101_636, 99_542_125, 0.7, 1024, 256, 2, 1, 100),
    # [2] PubMed-shaped, K = 1024 (the metric's workload)
    "pubmed": CorpusConfig("pubmed", 8_200_000, 141_043, 737_869_083, 0.5, 1024, 256, 3, 1, 100),
    # [3] NYTimes-shaped K sweep
    "nytimes_k128": CorpusConfig("nytimes_k128", 299_752, 101_636, 99_542_125, 0.7, 128, 256, 2, 1, 100),
    "nytimes_k8192": CorpusConfig("nytimes_k8192", 299_752, 101_636, 99_542_125, 0.7, 8192, 256, 2, 1, 100),
    # [4] scaled PubMed, 8 GPUs
    "pubmed_x5": CorpusConfig("pubmed_x5", 44_400_000, 141_043, 4_000_000_000, 0.5, 1024, 256, 4, 1, 20),
}


def scaled(cfg: CorpusConfig, frac: float, name: str | None = None) -> CorpusConfig:
    """Same shape parameters, fewer docs/tokens (vocabulary kept)."""
    D = max(1, int(round(cfg.D * frac)))
    T = max(D, int(round(cfg.T * frac)))
    return CorpusConfig(name or f"{cfg.name}@{frac:g}", D, cfg.V, T, cfg.sigma, cfg.K,
                        cfg.K_gen, cfg.corpus_seed, cfg.seed, cfg.sweeps)


def _doc_lengths(D, T, sigma, g, dev):
    if T < D:
        raise ValueError("need T >= D (every doc has >= 1 token)")
    mu = math.log(T / D) - 0.5 * sigma * sigma
    L = torch.exp(mu + sigma * torch.randn(D, generator=g, device=dev, dtype=torch.float64))
    L = L.round().clamp_(1, 65535).to(torch.int64)
    diff = int(T - int(L.sum()))
    while diff != 0:
        if diff > 0:
            idx = torch.randint(0, D, (diff,), generator=g, device=dev)
            L += torch.bincount(idx, minlength=D)
            L.clamp_(max=65535)
        else:
            idx = torch.randint(0, D, (min(-diff, D),), generator=g, device=dev)
            dec = torch.minimum(torch.bincount(idx, minlength=D), L - 1)
            L -= dec
        diff = int(T - int(L.sum()))
    return L


def _inverse_cdf_rows(weights):
    """Row-wise CDF with the last entry forced to exactly 1."""
    cdf = torch.cumsum(weights / weights.sum(dim=1, keepdim=True), dim=1)
    cdf[:, -1] = 1.0
    return cdf


def generate(D, V, T, sigma=0.5, K_gen=16, corpus_seed=1, device="cpu",
             alpha_gen=0.1, eta_scale=0.1, zipf_s=1.0, doc_chunk=200_000):
    """Returns (doc_ptr int64[D+1], words int32[T], z_true uint16[T]) as torch
    tensors on ``device``."""
    dev = torch.device(device)
    g = torch.Generator(device=dev)
    g.manual_seed(int(corpus_seed))
    f64 = torch.float64
    L = _doc_lengths(D, T, sigma, g, dev)
    doc_ptr = torch.zeros(D + 1, dtype=torch.int64, device=dev)
    torch.cumsum(L, 0, out=doc_ptr[1:])

    pi = torch.arange(1, V + 1, device=dev, dtype=f64).pow(-zipf_s)
    pi /= pi.sum()
    conc = (eta_scale * V * pi).unsqueeze(0).expand(K_gen, V).contiguous()
    phi = torch._standard_gamma(conc, generator=g)
    phi_flat = (_inverse_cdf_rows(phi) + torch.arange(K_gen, device=dev, dtype=f64)[:, None]).reshape(-1)
    del phi, conc

    words = torch.empty(T, dtype=torch.int32, device=dev)
    z_true = torch.empty(T, dtype=torch.int16, device=dev)
    a_gen = torch.full((1, K_gen), alpha_gen, dtype=f64, device=dev)
    for d0 in range(0, D, doc_chunk):
        d1 = min(D, d0 + doc_chunk)
        nd = d1 - d0
        theta = torch._standard_gamma(a_gen.expand(nd, K_gen).contiguous(), generator=g)
        theta_flat = (_inverse_cdf_rows(theta) + torch.arange(nd, device=dev, dtype=f64)[:, None]).reshape(-1)
        t0, t1 = int(doc_ptr[d0]), int(doc_ptr[d1])
        local_doc = torch.repeat_interleave(torch.arange(nd, device=dev, dtype=torch.int64), L[d0:d1])
        u = torch.rand(t1 - t0, generator=g, device=dev, dtype=f64)
        z = torch.searchsorted(theta_flat, u + local_doc.to(f64), right=True) - local_doc * K_gen
        z.clamp_(0, K_gen - 1)
        u2 = torch.rand(t1 - t0, generator=g, device=dev, dtype=f64)
        w = torch.searchsorted(phi_flat, u2 + z.to(f64), right=True) - z * V
        w.clamp_(0, V - 1)
        words[t0:t1] = w.to(torch.int32)
        z_true[t0:t1] = z.to(torch.int16)
        del theta, theta_flat, local_doc, u, z, u2, w
    return doc_ptr, words, z_true   # z_true: int16 bit pattern of uint16


def generate_config(cfg: CorpusConfig, device="cpu"):
    return generate(cfg.D, cfg.V, cfg.T, cfg.sigma, cfg.K_gen, cfg.corpus_seed, device)


def to_numpy(doc_ptr, words, z_true=None):
    out = [doc_ptr.cpu().numpy().astype(np.int64, copy=False),
           words.cpu().numpy().astype(np.int32, copy=False)]
    if z_true is not None:
        out.append(z_true.cpu().view(torch.int16).numpy().view(np.uint16))
    return tuple(out)


def tiny_numpy():
    """The tiny config (BASELINE.json configs[0]) as numpy arrays."""
    cfg = CONFIGS["tiny"]
    return to_numpy(*generate_config(cfg, "cpu"))
