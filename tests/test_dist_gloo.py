"""The multi-GPU decomposition on CPU (-m "not gpu"): world_size 2 over gloo.

Each rank owns a token-balanced contiguous document range (the library's
lda_partition_docs, X21), computes its canonical-index bases from the
all-gathered word histograms (the library's lda_canonical_bases, the
arithmetic lda_load_corpus runs before its NCCL path), draws its documents'
tokens against the replicated global counts (the oracle's per-document draw),
and sum-allreduces its partial counts (Eq. 4).  The result must be
bit-identical to one process running the whole sweep.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

WORLD = 2


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, out_q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_hpdc_xie0lt19_b200 as L
        from oracle import oracle as O
        from paper_conf_hpdc_xie0lt19_b200 import synth

        c = synth.CONFIGS["tiny"]
        doc_ptr, words, _ = synth.tiny_numpy()
        D, V, K = c.D, c.V, c.K
        bounds = L.lda_partition_docs(doc_ptr, world)
        d0, d1 = int(bounds[rank]), int(bounds[rank + 1])
        t0, t1 = int(doc_ptr[d0]), int(doc_ptr[d1])

        # canonical bases from all-gathered per-rank word histograms
        local = torch.from_numpy(np.bincount(words[t0:t1], minlength=V).astype(np.int64))
        gathered = [torch.zeros(V, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(gathered, local)
        cbase, T = L.lda_canonical_bases(torch.stack(gathered).numpy(), rank)
        seen = np.zeros(V, np.int64)
        my_canon = np.empty(t1 - t0, np.int64)
        for i in range(t0, t1):
            w = words[i]
            my_canon[i - t0] = cbase[w] + seen[w]
            seen[w] += 1
        canon = O.canonical_order(doc_ptr, words, V)
        ok_canon = bool(np.array_equal(my_canon, canon[t0:t1])) and T == len(words)

        # three synchronous sweeps, each rank drawing only its documents
        z = np.empty(len(words), np.uint16)
        O.lib().orc_init(len(words), canon, K, c.seed, z)
        nwk = np.zeros(V * K, np.int32)
        nk = np.zeros(K, np.int32)
        ndk = np.zeros(D * K, np.int32)
        O.lib().orc_counts(D, V, K, doc_ptr, words, z, nwk, nk, ndk.ctypes.data_as(O.ctypes.c_void_p))
        for t in (1, 2, 3):
            zn = O.draw_docs(d0, d1, doc_ptr, words, canon, V, K, c.alpha, c.beta, c.seed, t, z, nwk,
                             nk, ndk)
            part = np.zeros((V, K), np.int64)
            np.add.at(part, (words[t0:t1], zn[t0:t1].astype(np.int64)), 1)
            tot = torch.from_numpy(part.reshape(-1))
            dist.all_reduce(tot)                       # ϕ = Σ_g ϕ_g  (Eq. 4)
            zsum = torch.from_numpy(zn.astype(np.int64))
            dist.all_reduce(zsum)                      # each rank filled only its docs
            z = zsum.numpy().astype(np.uint16)
            nwk = tot.numpy().astype(np.int32)
            nk = nwk.reshape(V, K).sum(0).astype(np.int32)
            d = np.repeat(np.arange(D), np.diff(doc_ptr))
            ndk = np.zeros((D, K), np.int32)
            np.add.at(ndk, (d, z.astype(np.int64)), 1)
            ndk = ndk.reshape(-1)
        out_q.put((rank, ok_canon, z.tobytes(), nwk.tobytes(), (d0, d1)))
    finally:
        dist.destroy_process_group()


@pytest.mark.timeout(600)
def test_two_rank_sweeps_equal_single_process():
    from oracle import oracle as O
    from paper_conf_hpdc_xie0lt19_b200 import synth

    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, WORLD, port, q)) for r in range(WORLD)]
    for p in procs:
        p.start()
    res = [q.get(timeout=540) for _ in range(WORLD)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    res.sort()

    c = synth.CONFIGS["tiny"]
    doc_ptr, words, _ = synth.tiny_numpy()
    ref = O.OracleLDA(c.D, c.V, c.K, c.alpha, c.beta).load(doc_ptr, words, c.seed)
    ref.iterate(3)
    ranges = [r[4] for r in res]
    assert ranges[0][0] == 0 and ranges[-1][1] == c.D and ranges[0][1] == ranges[1][0]
    for rank, ok_canon, zb, nwkb, _ in res:
        assert ok_canon, f"rank {rank}: canonical bases disagree with the global order"
        assert np.array_equal(np.frombuffer(zb, np.uint16), ref.z)
        assert np.array_equal(np.frombuffer(nwkb, np.int32), ref.n_wk)
