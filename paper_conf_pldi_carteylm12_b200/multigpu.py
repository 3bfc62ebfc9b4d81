"""Batch sharding across the GPUs of one box (the paper's `map`,
PAPER.md L194–L195, with one problem per multiprocessor, L407–L409).

Problems are independent, so there is no data-path collective: every rank
solves its shard with the CUDA library, then one gather puts the scores (and,
optionally, the tracebacks) back in input order. `torch.distributed` supplies
the process group (NCCL on the B200 box, gloo in the CPU tests).

Shards:
  * contiguous equal blocks for equal-cost problems (alignment, HMM);
  * cost-balanced "snake" dealing of the length-sorted problems for Nussinov,
    whose cost grows as n^3 — the permutation is kept to restore input order.
"""
from __future__ import annotations

import numpy as np


def shard_contiguous(n: int, world: int, rank: int) -> np.ndarray:
    """Ids of rank's contiguous block (sizes differ by at most one)."""
    base, extra = divmod(n, world)
    start = rank * base + min(rank, extra)
    return np.arange(start, start + base + (1 if rank < extra else 0), dtype=np.int64)


def shard_by_cost(costs, world: int, rank: int) -> np.ndarray:
    """Deal problems sorted by decreasing cost in snake order 0..W-1, W-1..0, ..."""
    costs = np.asarray(costs)
    order = np.argsort(-costs, kind="stable")
    r = np.arange(len(order))
    cyc = r % (2 * world)
    owner = np.where(cyc < world, cyc, 2 * world - 1 - cyc)
    return np.sort(order[owner == rank]).astype(np.int64)


def subset(cat, off, ids):
    """Packed sub-batch (cat, off) of the problems `ids`."""
    off = np.asarray(off)
    lens = off[ids + 1] - off[ids]
    new_off = np.zeros(len(ids) + 1, dtype=np.int64)
    np.cumsum(lens, out=new_off[1:])
    out = np.empty(int(new_off[-1]), dtype=np.uint8)
    for k, i in enumerate(ids):
        out[new_off[k]:new_off[k + 1]] = cat[off[i]:off[i + 1]]
    return out, new_off


def gather_in_order(local, ids, n_total, group=None, device=None):
    """All ranks contribute (ids, values); every rank gets the n_total values in input order.

    local: 1-D or 2-D torch tensor (rows = problems); ids: int64 numpy array."""
    import torch
    import torch.distributed as dist
    world = dist.get_world_size(group)
    dev = local.device if device is None else device
    counts = torch.tensor([len(ids)], dtype=torch.int64, device=dev)
    all_counts = [torch.zeros_like(counts) for _ in range(world)]
    dist.all_gather(all_counts, counts, group=group)
    m = int(max(int(c.item()) for c in all_counts))
    pad_shape = (m,) + tuple(local.shape[1:])
    buf = torch.zeros(pad_shape, dtype=local.dtype, device=dev)
    buf[:len(ids)] = local
    idb = torch.full((m,), -1, dtype=torch.int64, device=dev)
    idb[:len(ids)] = torch.as_tensor(ids, dtype=torch.int64, device=dev)
    vals = [torch.zeros_like(buf) for _ in range(world)]
    idss = [torch.zeros_like(idb) for _ in range(world)]
    dist.all_gather(vals, buf, group=group)
    dist.all_gather(idss, idb, group=group)
    out = torch.zeros((n_total,) + tuple(local.shape[1:]), dtype=local.dtype, device=dev)
    for v, i in zip(vals, idss):
        keep = i >= 0
        out[i[keep]] = v[keep]
    return out


def solve_sharded(solve_fn, a_cat, a_off, b_cat=None, b_off=None, *, by_cost=False, group=None, device=None):
    """Shard a host batch over the ranks of `group`, run `solve_fn(a_cat, a_off, b_cat, b_off) -> tensor`
    on this rank's shard, and return all scores in input order on every rank."""
    import torch.distributed as dist
    world, rank = dist.get_world_size(group), dist.get_rank(group)
    n = len(a_off) - 1
    if by_cost:
        lens = np.diff(np.asarray(a_off))
        ids = shard_by_cost(lens.astype(np.float64) ** 3, world, rank)
    else:
        ids = shard_contiguous(n, world, rank)
    sa, so = subset(a_cat, a_off, ids)
    sb = sbo = None
    if b_cat is not None:
        sb, sbo = subset(b_cat, b_off, ids)
    local = solve_fn(sa, so, sb, sbo)
    return gather_in_order(local, ids, n, group=group, device=device)
