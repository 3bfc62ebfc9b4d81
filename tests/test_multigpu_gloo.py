"""Multi-process host logic of the batch sharding on CPU with the
gloo backend, world size 2. The per-rank GPU solve is stood in for by the
oracle (the shards and the order-restoring gather are what is under test)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import dpgen
from paper_conf_pldi_carteylm12_b200 import multigpu


def test_shard_partitions():
    for n, w in [(10, 3), (100_000, 8), (7, 8), (0, 2)]:
        ids = np.concatenate([multigpu.shard_contiguous(n, w, r) for r in range(w)])
        assert (np.sort(ids) == np.arange(n)).all()
    costs = np.random.default_rng(0).integers(128, 513, size=1000) ** 3
    parts = [multigpu.shard_by_cost(costs, 4, r) for r in range(4)]
    assert sorted(np.concatenate(parts).tolist()) == list(range(1000))
    loads = [costs[p].sum() for p in parts]
    assert max(loads) / min(loads) < 1.02   # snake dealing balances n^3 work


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import oracle
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        # Nussinov batch with ragged lengths (cost-sharded) and an SW batch (contiguous)
        ids = dpgen.config5_sample_ids(n_seqs=10_000, k=37)
        cat, off = dpgen.config5_rna_batch(n_seqs=10_000, lo=20, hi=90, ids=ids)

        def nuss(a, o, b, bo):
            return torch.as_tensor(oracle.nussinov_batch(a, o, dpgen.rna_pair_mask(), 3), dtype=torch.int32)

        got = multigpu.solve_sharded(nuss, cat, off, by_cost=True)
        a_cat, a_off, b_cat, b_off = dpgen.config2_protein_pairs(21, 40)

        def sw(a, o, b, bo):
            return torch.as_tensor(oracle.sw_batch(a, o, b, bo, dpgen.blosum62(), 4), dtype=torch.int32)

        got_sw = multigpu.solve_sharded(sw, a_cat, a_off, b_cat, b_off)
        if rank == 0:
            q.put((got.numpy().tolist(), got_sw.numpy().tolist()))
    finally:
        dist.destroy_process_group()


def test_sharded_gather_matches_single_process():
    import oracle
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    nuss, swv = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    ids = dpgen.config5_sample_ids(n_seqs=10_000, k=37)
    cat, off = dpgen.config5_rna_batch(n_seqs=10_000, lo=20, hi=90, ids=ids)
    assert nuss == oracle.nussinov_batch(cat, off, dpgen.rna_pair_mask(), 3).tolist()
    a_cat, a_off, b_cat, b_off = dpgen.config2_protein_pairs(21, 40)
    assert swv == oracle.sw_batch(a_cat, a_off, b_cat, b_off, dpgen.blosum62(), 4).tolist()


def _bench_worker(rank, world, port, q):
    """bench.py's own shard + gather code (shard_ids, subset, Gatherer) with the oracle as the
    per-rank solve: scores and traceback rows come back in input order on every rank."""
    import bench
    import oracle
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        pm = dpgen.rna_pair_mask()
        # Nussinov: ragged lengths, the n^3 snake deal (non-contiguous shards)
        lens = dpgen.rng(6).integers(20, 90, size=41)
        seqs = [dpgen.random_seq(dpgen.rng(6, extra=k + 1), int(l), 4) for k, l in enumerate(lens)]
        cat, off = dpgen.pack(seqs)
        ids = bench.shard_ids("nuss5", len(seqs), np.diff(off), rank, world, "strong")
        scat, soff = bench.subset(cat, off, ids)
        sc = np.zeros(len(ids), np.int32)
        tb = np.zeros((len(ids), 96), np.uint8)
        tl = np.zeros(len(ids), np.int32)
        for k in range(len(ids)):
            v, db = oracle.nussinov_traceback(scat[soff[k]:soff[k + 1]], pm, 3)
            sc[k], tl[k] = v, len(db)
            tb[k, :len(db)] = np.frombuffer(db.encode(), np.uint8)
        g = bench.Gatherer(ids, len(seqs), torch.device("cpu"))
        got = (g("s", torch.from_numpy(sc)).numpy().tolist(), g("tb", torch.from_numpy(tb)).numpy(),
               g("tl", torch.from_numpy(tl)).numpy().tolist(), g.contiguous)
        # SW: contiguous blocks of the config-2 stream
        n = 23
        sids = bench.shard_ids("sw", n, None, rank, world, "strong")
        a_cat, a_off, b_cat, b_off = dpgen.config2_protein_pairs(n, 40)
        a_cat, a_off2 = bench.subset(a_cat, a_off, sids)
        b_cat, b_off = bench.subset(b_cat, b_off, sids)
        a_off = a_off2
        s2 = torch.as_tensor(oracle.sw_batch(a_cat, a_off, b_cat, b_off, dpgen.blosum62(), 4), dtype=torch.int32)
        g2 = bench.Gatherer(sids, n, torch.device("cpu"))
        got_sw = (g2("s", s2).numpy().tolist(), g2.contiguous)
        if rank == 0:
            q.put((got, got_sw, len(ids)))
    finally:
        dist.destroy_process_group()


def test_bench_shard_and_gather_world2():
    import oracle
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_bench_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    (sc, tb, tl, contig), (sw, contig_sw), n0 = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    assert not contig and contig_sw and 0 < n0 < 41
    pm = dpgen.rna_pair_mask()
    lens = dpgen.rng(6).integers(20, 90, size=41)
    for k, l in enumerate(lens):
        x = dpgen.random_seq(dpgen.rng(6, extra=k + 1), int(l), 4)
        v, db = oracle.nussinov_traceback(x, pm, 3)
        assert sc[k] == v and tl[k] == len(db) and bytes(tb[k, :tl[k]]).decode() == db
    a_cat, a_off, b_cat, b_off = dpgen.config2_protein_pairs(23, 40)
    assert sw == oracle.sw_batch(a_cat, a_off, b_cat, b_off, dpgen.blosum62(), 4).tolist()


def test_bench_subset_matches_python_loop():
    import bench
    g = np.random.default_rng(5)
    seqs = [g.integers(0, 4, size=int(g.integers(0, 30))).astype(np.uint8) for _ in range(50)]
    cat, off = dpgen.pack(seqs)
    ids = np.sort(g.choice(50, 17, replace=False))
    a, o = bench.subset(cat, off, ids)
    b, p = multigpu.subset(cat, off, ids)
    assert (a == b).all() and (o == p).all()
