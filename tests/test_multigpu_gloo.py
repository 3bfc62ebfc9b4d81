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
