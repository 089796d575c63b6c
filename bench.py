#!/usr/bin/env python
"""Throughput of the LDA collapsed-Gibbs sweep (CuLDA_CGS hot path) on B200.

Metric (BASELINE.json): tokens sampled per second per sweep (Eq. 2, PAPER.md
L427-433: #Tokens × #Iterations / ElapsedTime) on the PubMed-shaped synthetic
corpus (Table 3 shape, L1361-1363) at K = 1024, plus the HBM-roofline
fraction of the dominant kernel.  A "step" is one sweep (all §8(a) rows:
prologue, sampling, n_wk/n_k recount, θ rebuild, and the n_wk allreduce when
N > 1).

  python bench.py [--gpus N --steps K --warmup W] [--config pubmed]
  python bench.py --impl reference ...     # the CPU oracle on a bounded sample

One process per GPU (torchrun for N > 1): documents are partitioned by tokens
(lda_partition_docs), n_wk/n_k are sum-allreduced every sweep over NCCL;
total work is fixed as N grows ("scaling": "strong").  Inputs (GBs) are far
larger than the 126 MB L2, so no L2 flush is needed between steps.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

FALLBACK_HBM_GBS = 6650.0  # /opt/skills/guides/B200_PROFILING.md fallback


def _peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return float(p["hbm_gbs"]), "measured"
    except Exception:
        return FALLBACK_HBM_GBS, "fallback"


class ClockSampler:
    """SM clocks + throttle reasons sampled during the timed region, in
    process through NVML (no subprocess: a fork of this process, which holds
    GBs of pinned host memory, could stall the launching thread inside the
    timed region); nvidia-smi only when NVML is unavailable."""

    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.rows = []
        self._stop = threading.Event()
        self._t = None

    def _nvml_rows(self):
        import pynvml as N
        N.nvmlInit()
        try:
            h = N.nvmlDeviceGetHandleByIndex(int(self.index))
            bits = (N.nvmlClocksEventReasonHwSlowdown, N.nvmlClocksEventReasonHwThermalSlowdown,
                    N.nvmlClocksEventReasonSwThermalSlowdown, N.nvmlClocksEventReasonSwPowerCap)
            while not self._stop.is_set():
                sm = N.nvmlDeviceGetClockInfo(h, N.NVML_CLOCK_SM)
                mx = N.nvmlDeviceGetMaxClockInfo(h, N.NVML_CLOCK_SM)
                r = N.nvmlDeviceGetCurrentClocksEventReasons(h)
                self.rows.append([str(sm), str(mx), ""] + ["Active" if r & b else "Not Active" for b in bits])
                self._stop.wait(0.05)
        finally:
            N.nvmlShutdown()

    def _run(self):
        try:
            self._nvml_rows()
            return
        except Exception:
            pass
        while not self._stop.is_set():
            try:
                out = subprocess.run(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                      "--format=csv,noheader,nounits"], capture_output=True, text=True,
                                     timeout=5).stdout.strip()
                if out:
                    self.rows.append([x.strip() for x in out.split(",")])
            except Exception:
                pass
            self._stop.wait(0.1)

    def __enter__(self):
        self._t = threading.Thread(target=self._run, daemon=True)
        self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        self._t.join(timeout=10)

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"], "samples": 0}
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4) if len(r) > 3 + i and r[3 + i] == "Active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows)}


def _dist():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


# ---------------------------------------------------------------------------
# CPU oracle legs (the only places bench.py executes oracle/)
# ---------------------------------------------------------------------------

def _oracle_sample(cfg, frac):
    from paper_conf_hpdc_xie0lt19_b200 import synth
    sub = synth.scaled(cfg, frac)
    doc_ptr, words = synth.to_numpy(*synth.generate_config(sub, "cpu"))[:2]
    return sub, doc_ptr, words


def cpu_oracle_rate(cfg, budget_s=20.0, frac=None, start_sweep=1, warm_budget_s=12.0):
    """Time the oracle (as it stands, one thread) on a doc-prefix-shaped
    sample of the workload, at the GPU's sweep index: the sample is first
    advanced to sweep start_sweep - 1 by oracle-omp (bit-identical, all host
    cores, untimed, bounded by warm_budget_s), then single-threaded sweeps
    are timed; returns tokens/s of the timed sweeps."""
    from oracle import oracle as O
    frac = frac if frac is not None else max(2e-4, min(1.0, 0.75e6 / cfg.T))
    sub, doc_ptr, words = _oracle_sample(cfg, frac)
    m = O.OracleLDA(sub.D, sub.V, sub.K, sub.alpha, sub.beta).load(doc_ptr, words, sub.seed)
    tw = time.perf_counter()
    while m.t < start_sweep - 1 and time.perf_counter() - tw < warm_budget_s:
        m.iterate(1, parallel=True)
    first = m.t + 1
    toks, secs, sweeps = 0, 0.0, 0
    while (secs < budget_s or sweeps == 0) and sweeps < 100:
        t0 = time.perf_counter()
        m.iterate(1)
        secs += time.perf_counter() - t0
        toks += sub.T
        sweeps += 1
    return toks / secs, {"docs": sub.D, "tokens": sub.T, "sweeps": [first, first + sweeps - 1],
                         "seconds": round(secs, 3), "frac_of_corpus": frac, "omp_threads": O.omp_threads()}


def run_reference(args):
    rank, world, _ = _dist()
    if rank != 0:
        return 0
    from paper_conf_hpdc_xie0lt19_b200 import synth
    cfg = synth.CONFIGS[args.config]
    # size the per-step sample so warmup+steps take ~120 s in total
    rate, _ = cpu_oracle_rate(cfg, budget_s=3.0, frac=max(2e-4, 0.05e6 / cfg.T))
    per_step_tokens = max(20_000, rate * 120.0 / max(1, args.steps + args.warmup))
    frac = min(1.0, per_step_tokens / cfg.T)
    from oracle import oracle as O
    sub, doc_ptr, words = _oracle_sample(cfg, frac)
    m = O.OracleLDA(sub.D, sub.V, sub.K, sub.alpha, sub.beta).load(doc_ptr, words, sub.seed)
    for _ in range(args.warmup):
        m.iterate(1)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        m.iterate(1)
    dt = time.perf_counter() - t0
    value = sub.T * args.steps / dt
    sample = (f"oracle (single-threaded C, fp64) SWEEP mode on a {cfg.name}-shaped corpus of "
              f"{sub.D} docs / {sub.T} tokens (frac {frac:.3g} of the full workload, same V, K, shape)")
    line = {"impl": "reference", "metric": "tokens sampled/sec per sweep", "value": value,
            "unit": "tokens/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": 1e3 * dt / args.steps, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": cfg.name, "D": cfg.D, "V": cfg.V, "T": cfg.T, "K": cfg.K,
                       "alpha": cfg.alpha, "beta": cfg.beta, "sample_tokens": sub.T},
            "cpu_baseline": {"value": value, "unit": "tokens/s", "cores": 1, "kind": "oracle",
                             "sample": sample},
            "e2e": {"value": value, "unit": "tokens/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


# ---------------------------------------------------------------------------
# the CUDA path
# ---------------------------------------------------------------------------

def run_b200(args):
    import torch
    import torch.distributed as dist

    import paper_conf_hpdc_xie0lt19_b200 as L
    from paper_conf_hpdc_xie0lt19_b200 import config as C
    from paper_conf_hpdc_xie0lt19_b200 import synth

    rank, world, local = _dist()
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    cfg = synth.CONFIGS[args.config]
    dev = torch.device("cuda", local)

    # ---- synthetic corpus (untimed), same on every rank; each keeps its docs
    t_gen = time.perf_counter()
    doc_ptr_t, words_t, _ = synth.generate_config(cfg, dev)
    doc_ptr_full = doc_ptr_t.cpu().numpy()
    bounds = L.lda_partition_docs(doc_ptr_full, world)
    d0, d1 = int(bounds[rank]), int(bounds[rank + 1])
    t0_, t1_ = int(doc_ptr_full[d0]), int(doc_ptr_full[d1])
    words = torch.empty(t1_ - t0_, dtype=torch.int32, pin_memory=True)
    words.copy_(words_t[t0_:t1_])
    words = words.numpy()
    doc_ptr = (doc_ptr_full[d0:d1 + 1] - t0_).astype(np.int64)
    del doc_ptr_t, words_t
    torch.cuda.empty_cache()
    t_gen = time.perf_counter() - t_gen

    uid = None
    if world > 1:
        obj = [L.lda_nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        uid = obj[0]

    opts = {}   # the library's defaults; --opt only for experiments
    for kv in args.opt:
        k, v = kv.split("=")
        opts[k] = int(v)

    def make_model():
        m = L.LDA(cfg.D, cfg.V, cfg.K, cfg.alpha, cfg.beta, device=local, **opts)
        if world > 1:
            m.init_dist(rank, world, uid)
        return m

    def barrier():
        if world > 1:
            dist.barrier(device_ids=[local])
        torch.cuda.synchronize()

    # ---- end to end through the public API with host buffers:
    #      load (H2D + prep + init) + K sweeps + D2H of z, wall clock.
    #      Inputs and the z output live in pinned host memory (allocated
    #      before the timed region, like the input staging).
    z_pinned = torch.empty(t1_ - t0_, dtype=torch.int16, pin_memory=True).numpy().view(np.uint16)
    barrier()
    te0 = time.perf_counter()
    m = make_model()
    m.load(doc_ptr, words, cfg.seed, d0, d1)
    te1 = time.perf_counter()
    m.iterate(args.steps)
    te2 = time.perf_counter()
    z_host = m.z(out=z_pinned)
    barrier()
    te = time.perf_counter() - te0
    e2e_parts = {"create_load_s": round(te1 - te0, 3), "iterate_s": round(te2 - te1, 3),
                 "z_d2h_s": round(te0 + te - te2, 3)}
    e2e_times = torch.tensor([te], device=dev, dtype=torch.float64)
    if world > 1:
        dist.all_reduce(e2e_times, op=dist.ReduceOp.MAX)
    e2e_value = cfg.T * args.steps / float(e2e_times.item())
    h2d = (doc_ptr.nbytes + words.nbytes) / args.steps
    d2h = z_host.nbytes / args.steps

    # ---- device-timed: W warm-up sweeps, then exactly K timed sweeps
    m.iterate(args.warmup)
    stream = torch.cuda.ExternalStream(m.stream(), device=dev)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    idx = torch.cuda.current_device()
    phys = os.environ.get("CUDA_VISIBLE_DEVICES", str(idx)).split(",")[idx] if os.environ.get("CUDA_VISIBLE_DEVICES") else str(idx)
    barrier()
    with ClockSampler(phys) as clk:
        time.sleep(0.3)
        ev0.record(stream)
        m.iterate(args.steps)
        ev1.record(stream)
        barrier()
        time.sleep(0.2)
    ms = ev0.elapsed_time(ev1)
    st = m.stats()
    log = m.sweep_log()
    t = torch.tensor([ms, st["ms_sample"], st["ms_allreduce"], st["ms_theta"], st["ms_recount"],
                      st["ms_allreduce_exposed"]], device=dev, dtype=torch.float64)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms_max = float(t[0])
    value = cfg.T * args.steps / (ms_max / 1e3)

    # roofline of the dominant kernel (sampling), SURVEY §8(d) byte model
    peak, peak_src = _peaks()
    T_g, D_g = int(doc_ptr[-1]), d1 - d0
    b_sample = sum(C.bytes_sample(T_g, cfg.V, cfg.K, int(n)) for n in log["sum_nnz_tok"])
    # the sampling kernel alone: its events bracket the kernel on the library
    # stream (the per-word table kernel before it is reported separately)
    t_sample = (float(np.sum(log["ms_sample"])) - float(st["ms_table"])) / 1e3
    achieved = b_sample / t_sample / 1e9
    kernel = {2: "sweep_tile_kernel", 3: "sweep_tile_cta_kernel"}.get(int(st["sampler"]), "sweep_kernel")
    b_sweep = sum(C.bytes_sweep(T_g, D_g, cfg.V, cfg.K, int(a), int(b)) for a, b in
                  zip(log["sum_nnz_tok"], log["sum_nnz_doc"]))
    sweep_gbs = b_sweep / (float(np.sum(log["ms_sweep"])) / 1e3) / 1e9
    # DRAM bytes per launch of the sampling kernel from the committed ncu
    # capture of this config (profiles/traffic.json, tools/write_traffic.py)
    traffic, traffic_src = None, None
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
            tr = json.load(f).get(cfg.name)
        if tr:
            traffic = float(tr["sweep_kernel_dram_bytes_per_launch"])
            traffic_src = f"{tr['report']} ({tr['round']})"
    except Exception:
        pass
    t_sample_launch = t_sample / args.steps

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        first_timed = int(st["sweeps_done"]) - args.steps + 1
        rate, info = cpu_oracle_rate(cfg, budget_s=args.cpu_budget, start_sweep=first_timed)
        cpu = {"value": rate, "unit": "tokens/s", "cores": 1, "kind": "oracle",
               "sample": (f"oracle (single-threaded C, fp64) SWEEP mode, timed sweeps "
                          f"{info['sweeps'][0]}..{info['sweeps'][1]} (the GPU's timed window starts at "
                          f"{first_timed}; earlier sweeps by oracle-omp on {info['omp_threads']} threads, "
                          f"untimed) on a {cfg.name}-shaped corpus of {info['docs']} docs / "
                          f"{info['tokens']} tokens (frac {info['frac_of_corpus']:.3g}; same V, K, shape), "
                          f"{info['seconds']} s")}

    if rank == 0:
        clocks = clk.summary()
        mean_nnz = float(np.mean(log["sum_nnz_tok"])) / max(T_g, 1)
        line = {
            "metric": "tokens sampled/sec per sweep", "value": value, "unit": "tokens/s",
            "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": ms_max / args.steps, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": cfg.name, "D": cfg.D, "V": cfg.V, "T": cfg.T, "K": cfg.K,
                       "alpha": cfg.alpha, "beta": cfg.beta, "seed": cfg.seed,
                       "timed_sweeps": [int(st["sweeps_done"]) - args.steps + 1, int(st["sweeps_done"])],
                       "l2": "inputs (GBs) larger than the 126 MB L2; no flush",
                       "parallelism": f"doc-partitioned dp{world}", "options": opts,
                       "sampler": int(st["sampler"]), "tile_tokens": int(st["tile_tokens"]),
                       "tiles": int(st["n_tiles"])},
            "roofline": {"bound": "hbm", "kernel": kernel, "achieved": achieved, "peak": peak,
                         "unit": "GB/s", "frac": achieved / peak, "traffic": traffic,
                         "achieved_basis": "algorithmic bytes (SURVEY §8(d) B_sample, measured nnz) / "
                                           "kernel event time",
                         "peak_source": peak_src,
                         "frac_of_8TBs_spec": achieved / 8000.0,
                         "algorithmic_bytes_per_launch": b_sample / args.steps,
                         "dram_achieved": (traffic / t_sample_launch / 1e9) if traffic else None,
                         "dram_frac": (traffic / t_sample_launch / 1e9 / peak) if traffic else None,
                         "traffic_over_algorithmic": (traffic / (b_sample / args.steps)) if traffic else None,
                         "traffic_source": traffic_src,
                         "sweep_achieved": sweep_gbs, "sweep_frac": sweep_gbs / peak,
                         "sweep_frac_of_8TBs_spec": sweep_gbs / 8000.0,
                         "bytes_per_token_model": b_sample / (T_g * args.steps)},
            "phases_ms_per_step": {"sample": float(t[1]) / args.steps,
                                   "sampler_kernel": 1e3 * t_sample / args.steps,
                                   "word_tables": float(st["ms_table"]) / args.steps,
                                   "recount": float(t[4]) / args.steps,
                                   "theta": float(t[3]) / args.steps,
                                   "allreduce_raw": float(t[2]) / args.steps,
                                   "allreduce_exposed": float(t[5]) / args.steps},
            "nnz_per_token": mean_nnz,
            "exact_redraws_per_step": st["n_exact_redraws"] / args.steps,
            "per_sweep_ms": [round(x, 4) for x in log["ms_sweep"].tolist()],
            "clocks": clocks,
            "e2e": {"value": e2e_value, "unit": "tokens/s", "h2d_bytes_per_step": int(h2d),
                    "d2h_bytes_per_step": int(d2h), "breakdown": e2e_parts,
                    "what": "lda_create+lda_load_corpus(host arrays: H2D, prep, init)+lda_iterate(K)+z D2H"},
            "gpu_launches": int(st["n_launches"]),
            "cpu_baseline": cpu,
            "gen_s": round(t_gen, 2),
        }
        print(json.dumps(line), flush=True)
    m.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="b200", choices=["b200", "reference"])
    ap.add_argument("--config", default="pubmed")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-budget", type=float, default=15.0)
    ap.add_argument("--opt", action="append", default=[], help="extra lda_set_option key=value")
    args = ap.parse_args()
    if args.warmup < 3 and args.impl == "b200":
        print("warning: --warmup < 3 violates the timing rules", file=sys.stderr)
    if args.impl == "reference":
        return run_reference(args)
    return run_b200(args)


if __name__ == "__main__":
    sys.exit(main())
