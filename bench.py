#!/usr/bin/env python
"""Benchmark: DP cell-updates/s (GCUPS) on B200 with the roofline fraction of the
dominant kernel (BASELINE.json metric; DESIGN.md §4 "Measurement").

Headline (`value`, N = 1): BASELINE config 2 — 100k synthetic protein pairs of
length 256, Smith–Waterman (BLOSUM62, linear gap 4) on the anti-diagonal
schedule. A step = one pass of the whole hot path over one batch: the schedule
(plan) already derived, solve with traceback retention, the canonical traceback
of every pair and, at N > 1, the NCCL gather of scores and tracebacks back into
input order. The same line carries a `configs` block with every other BASELINE
config (1, 3, 4, 5) and the §8(f) NEXT workloads, each with its own value,
step time, roofline, e2e and cpu_baseline.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                  [--config sw|swa|swshort|nuss1|hmm|nuss4|nuss5|nussmid|diag|phmm] [--only]
                  [--scaling strong|weak]

Multi-GPU (the paper's `map`, L194–L195, one problem per
multiprocessor, L407–L409): one process per GPU. Launched by torchrun, or, when
WORLD_SIZE is unset and --gpus N > 1, bench.py relaunches itself under
torch.distributed.run with N ranks. Each batched config's FIXED batch is
sharded (strong scaling: contiguous blocks for SW / HMM, an n^3-cost snake deal
for Nussinov) and after compute one NCCL all-gather per output restores input
order on every rank; `result_sha256` (scores + tracebacks in input order) is
the same at every N. Single-table configs (1, 4) run as replicas. Ranks are
timed with CUDA events and the max over ranks is reported.
"""
from __future__ import annotations

import argparse
import hashlib
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

import dpgen  # noqa: E402

METRIC = "DP cell-updates/sec (GCUPS) at 1/2/4/8 B200 and fraction of roofline"
MEASURED_UBENCH = {  # profiles/ubench_r01.jsonl, lane-ops per SM clock on B200 (this pool)
    "viaddmnmx_s32": 64.0, "viaddmnmx_s16x2": 128.0, "ffma": 128.0, "lds_bytes": 128.0,
}
SMS = 148
ALL_CONFIGS = ["sw", "nuss1", "hmm", "nuss4", "nuss5", "swa", "swshort", "nussmid", "diag", "phmm"]
# configs in the `configs` block at N > 1: the batched ones (the others are single tables: replicas only)
SHARDED = {"sw", "hmm", "nuss5", "swa", "swshort", "diag", "phmm"}


def peaks():
    p = {"hbm_gbs": 6570.6, "sm_max_mhz": 1965.0, "bf16_tflops": 1590.0, "source": "fallback"}
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            m = json.load(f)
        p.update({"hbm_gbs": m["hbm_gbs"], "sm_max_mhz": m.get("sm_max_mhz", 1965.0),
                  "bf16_tflops": m.get("bf16_tflops", 1685.9), "source": "measured"})
    except Exception:
        pass
    return p


def traffic_table():
    """ncu dram__bytes_read.sum + dram__bytes_write.sum per launch of each dominant kernel, from one
    `ncu --set full` capture per config (profiles/traffic_r02.json; scripts/ncu_traffic.py)."""
    try:
        with open(os.path.join(ROOT, "profiles", "traffic_r02.json")) as f:
            return json.load(f)
    except Exception:
        return {}


# ----------------------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi clocks and throttle reasons sampled during the timed region."""

    def __init__(self, index):
        self.index = index
        self.samples = []
        self.proc = None

    def __enter__(self):
        q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={q}",
                                          "--format=csv,noheader,nounits", "-lms", "20"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.started = threading.Event()
            self.thread = threading.Thread(target=self._read, daemon=True)
            self.thread.start()
            self.started.wait(timeout=5.0)  # first sample (pre-region) is discarded
        except Exception:
            self.proc = None
        return self

    def _read(self):
        first = True
        for line in self.proc.stdout:
            parts = [x.strip() for x in line.split(",")]
            if len(parts) >= 6:
                if first:
                    first = False
                    self.started.set()
                    continue
                self.samples.append(parts)

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except Exception:
                self.proc.kill()

    def summary(self):
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"]}
        sm = [float(s[0]) for s in self.samples if s[0].replace(".", "").isdigit()]
        mx = [float(s[1]) for s in self.samples if s[1].replace(".", "").isdigit()]
        reasons = sorted({names[k] for s in self.samples for k in range(4) if s[2 + k].lower().startswith("active")})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.samples)}


# ----------------------------------------------------------------------------- sharding (host logic)
def shard_ids(name, n_total, lens, rank, world, scaling):
    """Global problem ids of this rank. Strong scaling shards the config's fixed
    batch: contiguous equal blocks (equal-cost problems) or, for Nussinov (cost ~ n^3), the snake
    deal of the cost-sorted problems. Weak scaling gives every rank a full batch of its own
    (ids offset by rank). Single-table configs are replicas."""
    from paper_conf_pldi_carteylm12_b200 import multigpu
    if world == 1 or name in ("nuss1", "nuss4"):
        return np.arange(n_total, dtype=np.int64)
    if scaling == "weak":
        return np.arange(n_total, dtype=np.int64) + rank * n_total
    if name == "nuss5":
        return multigpu.shard_by_cost(lens.astype(np.float64) ** 3, world, rank)
    return multigpu.shard_contiguous(n_total, world, rank)


def subset(cat, off, ids):
    """Packed sub-batch of the problems `ids` (vectorised)."""
    ids = np.asarray(ids, dtype=np.int64)
    lens = off[ids + 1] - off[ids]
    new_off = np.zeros(len(ids) + 1, dtype=np.int64)
    np.cumsum(lens, out=new_off[1:])
    if len(ids) == 0:
        return np.zeros(0, np.uint8), new_off
    src = np.repeat(off[ids] - new_off[:-1], lens) + np.arange(int(new_off[-1]), dtype=np.int64)
    return cat[src], new_off


class Gatherer:
    """The order-restoring gather after compute: every rank contributes its shard's
    rows (scores, and traceback rows + lengths); one all_gather_into_tensor per output (NCCL on the
    B200 box, gloo in the CPU test) of equal padded shards, then rows go back to input order. The
    problem ids are static, so they are gathered once at construction."""

    def __init__(self, ids, n_total, device):
        import torch
        import torch.distributed as dist
        self.world = dist.get_world_size()
        self.n = len(ids)
        t = torch.tensor([self.n], dtype=torch.int64, device=device)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        self.m = int(t.item())
        ids_pad = torch.full((self.m,), -1, dtype=torch.int64, device=device)
        ids_pad[:self.n] = torch.as_tensor(np.asarray(ids), dtype=torch.int64).to(device)
        all_ids = torch.empty(self.world * self.m, dtype=torch.int64, device=device)
        dist.all_gather_into_tensor(all_ids, ids_pad)
        self.keep = all_ids >= 0
        self.dst = all_ids[self.keep]
        self.n_total = n_total
        self.contiguous = bool((self.dst == torch.arange(n_total, device=device)).all().item())
        self.device = device
        self._bufs = {}

    def _buf(self, key, shape, dtype):
        import torch
        b = self._bufs.get(key)
        if b is None or b.shape != shape or b.dtype != dtype:
            b = self._bufs[key] = torch.zeros(shape, dtype=dtype, device=self.device)
        return b

    def __call__(self, key, local):
        """All rows of `local` (this rank's shard, n x ...) from every rank, in input order."""
        import torch.distributed as dist
        rest = tuple(local.shape[1:])
        pad = self._buf(("pad", key), (self.m,) + rest, local.dtype)
        big = self._buf(("big", key), (self.world * self.m,) + rest, local.dtype)
        pad[:self.n] = local
        dist.all_gather_into_tensor(big, pad)
        if self.contiguous:
            return big[self.keep]
        out = self._buf(("out", key), (self.n_total,) + rest, local.dtype)
        out[self.dst] = big[self.keep]
        return out


# ----------------------------------------------------------------------------- workloads
def workload(name, rank=0, world=1, scaling="strong"):
    """Host arrays of this rank's shard, plus the counts the metric and roofline use."""
    if name in ("sw", "swa"):
        n = 100_000
        if scaling == "weak" and world > 1:
            a_cat, a_off, b_cat, b_off = dpgen.config2_protein_pairs(n, 256, first=rank * n)
            ids = np.arange(n, dtype=np.int64) + rank * n
        else:   # the fixed batch, sliced (config2_protein_pairs' b rows depend on the total drawn)
            ids = shard_ids(name, n, None, rank, world, scaling)
            a_cat, a_off, b_cat, b_off = dpgen.config2_protein_pairs(n, 256)
            if world > 1:
                a_cat, a_off2 = subset(a_cat, a_off, ids)
                b_cat, b_off = subset(b_cat, b_off, ids)
                a_off = a_off2
        ops = 3 if name == "sw" else 6
        W = {"kind": name, "n_total": n, "ids": ids, "a_cat": a_cat, "a_off": a_off, "b_cat": b_cat, "b_off": b_off,
             "max_la": 256, "max_lb": 256, "cells_total": n * 65536, "cells_local": len(ids) * 65536,
             "ops_local": len(ids) * 65536 * ops, "tb_stride": 513}
        W["workload"] = ("BASELINE config 2: 100k protein pairs x 256 (uniform 20 aa), Smith-Waterman, BLOSUM62, "
                         "linear gap 4, with tracebacks" if name == "sw" else
                         "config 2 pairs with affine gaps (SURVEY 8(f) NEXT 1): 100k protein pairs x 256, "
                         "BLOSUM62, gap open 11 / extend 1, with tracebacks")
        return W
    if name in ("nuss1", "nuss4"):
        x = dpgen.config1_rna64() if name == "nuss1" else dpgen.config4_rna8192()
        n = len(x)
        cat, off = dpgen.pack([x])
        inner = n * (n - 1) * (n - 2) // 6
        return {"kind": "nuss", "config": name, "n_total": 1, "ids": np.zeros(1, np.int64), "a_cat": cat, "a_off": off,
                "max_la": n, "cells_total": n * (n - 1) // 2, "cells_local": n * (n - 1) // 2, "inner_local": inner,
                "tb_stride": n,
                "workload": ("BASELINE config 1: one 64-nt RNA, Nussinov (h=3, WC+GU), with traceback" if name == "nuss1"
                             else "BASELINE config 4: one 8192-nt RNA, Nussinov grid-wide hyperplane sweep, "
                                  "with traceback")}
    if name == "nussmid":
        cat, off = dpgen.mid_rna_batch()
        lens = np.diff(off)
        return {"kind": "nuss", "config": name, "n_total": len(lens), "ids": np.arange(len(lens), dtype=np.int64),
                "a_cat": cat, "a_off": off, "max_la": int(lens.max()),
                "cells_total": int((lens * (lens - 1) // 2).sum()), "cells_local": int((lens * (lens - 1) // 2).sum()),
                "inner_local": int((lens * (lens - 1) * (lens - 2) // 6).sum()), "tb_stride": int(lens.max()),
                "workload": "SURVEY 8(f) NEXT 4: 16 RNAs of length U[482,1024], Nussinov with tracebacks, one "
                            "thread-block cluster per problem (table in distributed shared memory)"}
    if name == "nuss5":
        nseq = int(os.environ.get("DP_NUSS5_N", 1_000_000))
        cat, off = dpgen.config5_rna_batch(nseq)
        lens_all = np.diff(off)
        ids = shard_ids(name, nseq, lens_all, rank, world, scaling) if scaling != "weak" else np.arange(nseq)
        if scaling == "weak" and world > 1:
            ids = np.arange(nseq, dtype=np.int64)  # weak: every rank folds the whole batch (same data)
        scat, soff = subset(cat, off, ids) if world > 1 else (cat, off)
        lens = np.diff(soff)
        return {"kind": "nuss", "config": name, "n_total": nseq, "ids": ids, "a_cat": scat, "a_off": soff,
                "max_la": int(lens_all.max()), "cells_total": int((lens_all * (lens_all - 1) // 2).sum()),
                "cells_local": int((lens * (lens - 1) // 2).sum()),
                "inner_local": int((lens * (lens - 1) * (lens - 2) // 6).sum()), "tb_stride": 512,
                "workload": "BASELINE config 5: 1M RNAs of length U[128,512], Nussinov batch, with tracebacks"}
    if name == "swshort":
        n = 1_000_000
        a_cat, a_off, b_cat, b_off = dpgen.short_protein_pairs(n)
        ids = shard_ids(name, n, None, rank, world, scaling)
        la, lb = np.diff(a_off), np.diff(b_off)
        if world > 1:
            a_cat, a_off2 = subset(a_cat, a_off, ids)
            b_cat, b_off2 = subset(b_cat, b_off, ids)
            a_off, b_off = a_off2, b_off2
        cells_local = int((np.diff(a_off) * np.diff(b_off)).sum())
        return {"kind": "swshort", "n_total": n, "ids": ids, "a_cat": a_cat, "a_off": a_off, "b_cat": b_cat,
                "b_off": b_off, "max_la": 64, "max_lb": 64, "cells_total": int((la * lb).sum()),
                "cells_local": cells_local, "ops_local": 3 * cells_local, "tb_stride": 129,
                "workload": "SURVEY 8(f) NEXT 1 (hybrid, short side): 1M protein pairs, |a| and |b| uniform in "
                            "[8, 64], Smith-Waterman, BLOSUM62, linear gap 4, with tracebacks (inter-task kernel)"}
    if name == "diag":
        n = 20_000
        a_cat, a_off, b_cat, b_off = dpgen.diag_pairs(n)
        ids = shard_ids(name, n, None, rank, world, scaling)
        la, lb = np.diff(a_off), np.diff(b_off)
        if world > 1:
            a_cat, a_off2 = subset(a_cat, a_off, ids)
            b_cat, b_off2 = subset(b_cat, b_off, ids)
            a_off, b_off = a_off2, b_off2
        return {"kind": "diag", "n_total": n, "ids": ids, "a_cat": a_cat, "a_off": a_off, "b_cat": b_cat,
                "b_off": b_off, "max_la": int(la.max()), "max_lb": int(lb.max()),
                "cells_total": int((la * lb).sum()), "cells_local": int((np.diff(a_off) * np.diff(b_off)).sum()),
                "ops_local": 3 * int((np.diff(a_off) * np.diff(b_off)).sum()), "tb_stride": None,
                "workload": "SURVEY 8(f) NEXT 2 (conditional schedules, §4.7): the diagonal-only recurrence "
                            "(longest common substring) over 20k DNA pairs, |a| and |b| log-uniform in "
                            "[32, 4096], schedule chosen per problem"}
    if name == "hmm":
        n = 10_000
        d = dpgen.config3_hmm(n_seqs=n)
        ids = shard_ids(name, n, None, rank, world, scaling)
        seqs = d["seqs"][ids]
        T = seqs.shape[1]
        off = np.arange(len(ids) + 1, dtype=np.int64) * T
        return {"kind": "hmm", "n_total": n, "ids": ids, "a_cat": seqs.reshape(-1).copy(), "a_off": off,
                "max_la": T, "hmm": d, "cells_total": 2 * n * 64 * T, "cells_local": 2 * len(ids) * 64 * T,
                "inner_local": len(ids) * 64 * 64 * (T - 1), "tb_stride": T,
                "workload": "BASELINE config 3: 64-state dense HMM, 10k DNA sequences x 1000, forward + Viterbi "
                            "with Viterbi tracebacks (cells = 2 tables x S x T x n)"}
    if name == "phmm":
        n = 13_355   # the database size of the paper's Fig.15 (L297)
        d = dpgen.profile_hmm_workload(n_seqs=n)
        ids = shard_ids(name, n, None, rank, world, scaling)
        cat, off = d["cat"], d["off"]
        if world > 1:
            cat, off = subset(cat, off, ids)
        lens = np.diff(off)
        L = d["L"]
        return {"kind": "phmm", "n_total": n, "ids": ids, "a_cat": cat, "a_off": off, "max_la": int(np.diff(d["off"]).max()),
                "phmm": d, "cells_total": int(3 * L * np.diff(d["off"]).sum()), "cells_local": int(3 * L * lens.sum()),
                "inner_local": int(L * lens.sum()), "tb_stride": None,
                "workload": f"SURVEY 8(f) NEXT 3: profile-HMM forward (§6.3), {L}-position protein profile, 13,355 "
                            f"sequences sampled from it (Fig.15's database size; cells = 3 tables x L x T)"}
    raise SystemExit(f"unknown config {name}")


# ----------------------------------------------------------------------------- our arm
def make_plans(dp, W):
    if W["kind"] in ("sw", "swshort"):
        return [dp.Plan(dp.SW_LINEAR, W["max_la"], W["max_lb"], sigma=dpgen.blosum62(), gap=dpgen.SW_GAP,
                        want_traceback=True)]
    if W["kind"] == "swa":
        return [dp.Plan(dp.SW_AFFINE, W["max_la"], W["max_lb"], sigma=dpgen.blosum62(), gap_open=dpgen.SW_GAP_OPEN,
                        gap_extend=dpgen.SW_GAP_EXTEND, want_traceback=True)]
    if W["kind"] == "diag":
        return [dp.Plan(dp.DIAG_LCS, W["max_la"], W["max_lb"], alphabet_size=4)]  # DNA
    if W["kind"] == "nuss":
        return [dp.Plan(dp.NUSSINOV, W["max_la"], pair_mask=dpgen.rna_pair_mask(), min_hairpin=dpgen.NUSS_HAIRPIN,
                        want_traceback=True)]
    if W["kind"] == "phmm":
        d = W["phmm"]
        return [dp.Plan(dp.PROFILE_FORWARD, W["max_la"], **d["model"])]
    h = W["hmm"]
    return [dp.Plan(dp.HMM_FORWARD, W["max_la"], pi=h["pi"], A=h["A"], E=h["E"]),
            dp.Plan(dp.HMM_VITERBI, W["max_la"], lpi=h["lpi"], lA=h["lA"], lE=h["lE"], want_traceback=True)]


PHASES = {
    "sw": ["k_sw16 (partition sweep)", "k_sw16_tb5 (traceback)"],
    "swshort": ["k_sw_inter (length sort + inter-task sweep)", "k_sw_inter_tb (traceback)"],
    "swa": ["k_align_affine (partition sweep)", "k_align_affine_tb (traceback)"],
    "nuss": ["k_nuss (fill + in-kernel traceback)", "dp_traceback (copy)"],
    "diag": ["k_diag (conditional schedule)"],
    "hmm": ["k_forward_tc (tcgen05 forward)", "k_viterbi16 (s16x2 max-plus, two sequences per register + fused path walk)", "k_viterbi_copy (traceback: path copy)"],
    "phmm": ["k_phmm_forward (anti-diagonal, three tables)"],
}


def run_config(name, args, rank, world, local_rank, steps, warmup, headline):
    import torch
    import torch.distributed as dist
    import paper_conf_pldi_carteylm12_b200 as dp

    dev = torch.device("cuda", local_rank)
    W = workload(name, rank, world, args.scaling)
    stream = torch.cuda.Stream(device=dev)

    def cu(x):
        return torch.from_numpy(np.ascontiguousarray(x)).to(dev)

    plans = make_plans(dp, W)
    dev_in = (cu(W["a_cat"]), cu(W["a_off"]), cu(W["b_cat"]) if "b_cat" in W else None,
              cu(W["b_off"]) if "b_off" in W else None)
    n = len(W["a_off"]) - 1
    fwd_like = W["kind"] in ("hmm", "phmm")
    scores = [torch.empty(n, dtype=torch.float32 if (fwd_like and k == 0) else torch.int32, device=dev)
              for k in range(len(plans))]
    tb_plan = plans[-1] if W["tb_stride"] else None
    stride = W["tb_stride"] or 0
    tb_out = torch.empty((n, stride), dtype=torch.uint8, device=dev)
    tb_len = torch.empty(n, dtype=torch.int32, device=dev)
    tb_co = torch.empty((n, 4), dtype=torch.int32, device=dev) if W["kind"] in ("sw", "swa", "swshort") else None
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)  # > 126 MB L2
    sharded = world > 1 and name in SHARDED and args.scaling == "strong"
    gat = Gatherer(W["ids"], W["n_total"], dev) if sharded else None
    final = {}

    phase_names = PHASES[W["kind"]][:len(plans) + (1 if tb_plan is not None else 0)]
    ev_phase = [[] for _ in phase_names]
    # the forward (79 latency-bound CTAs) on a HIGH-priority side stream: its CTAs are placed before
    # the Viterbi grid fills the SMs, and Viterbi takes every slot it leaves
    side = torch.cuda.Stream(device=dev, priority=-1) if W["kind"] == "hmm" else None

    def ev(st=None):
        e = torch.cuda.Event(enable_timing=True)
        e.record(st or stream)
        return e

    def gather():
        # all-gather every output (NCCL over NVLink), rows back in input order
        for k, sc in enumerate(scores):
            final[f"scores{k}"] = gat(f"scores{k}", sc)
        if tb_plan is not None:
            final["tb"] = gat("tb", tb_out)
            final["tl"] = gat("tl", tb_len)

    def step(timed):
        with torch.cuda.stream(stream), torch.cuda.nvtx.range(f"step {name}"):
            marks = [ev()] if timed else None
            if side is not None:
                # HMM: the forward (tensor cores) and Viterbi (ALU) are independent passes over the
                # same sequences: the forward on a side stream so Viterbi fills the SMs it leaves idle
                side.wait_event(ev())
                f0 = ev(side) if timed else None
                plans[0].solve_batch(*dev_in, max_len_a=W["max_la"], max_len_b=0, out=scores[0], stream=side)
                f1 = ev(side)
                if os.environ.get("DP_BENCH_VIT_DELAY"):  # experiment: let the forward's CTAs be placed first
                    torch.cuda._sleep(int(os.environ["DP_BENCH_VIT_DELAY"]))
                v0 = ev() if timed else None
                plans[1].solve_batch(*dev_in, max_len_a=W["max_la"], max_len_b=0, out=scores[1], stream=stream)
                if timed:
                    marks = [f0, f1, v0, ev()]
            else:
                for k, p in enumerate(plans):
                    p.solve_batch(*dev_in, max_len_a=W["max_la"], max_len_b=W.get("max_lb", 0), out=scores[k],
                                  stream=stream)
                    if timed:
                        marks.append(ev())
            if tb_plan is not None:
                tb_plan.traceback_into(0, n, tb_out, stride, tb_len, tb_co, stream=stream)
            if side is not None:
                stream.wait_event(f1)
            if timed:
                if tb_plan is not None:
                    marks.append(ev())
                if side is not None:  # forward, Viterbi, traceback (the first two overlap)
                    pairs = [(marks[0], marks[1]), (marks[2], marks[3]), (marks[3], marks[4])]
                else:
                    pairs = [(marks[q], marks[q + 1]) for q in range(len(phase_names))]
                for q in range(len(phase_names)):
                    ev_phase[q].append(pairs[q])
            if sharded:
                with torch.cuda.nvtx.range("gather (NCCL all-gather, input order)"):
                    gather()

    for _ in range(warmup):
        step(False)
    torch.cuda.synchronize(dev)
    W["variant"] = plans[0].last_variant  # the kernel family the plan dispatched to
    if W["kind"] == "swa" and W["variant"] == "k_affine16":
        phase_names = ["k_affine16 (packed s16x2 partition sweep)", "k_affine16_tb (traceback)"]
    launches0 = sum(p.launches for p in plans)
    step_ms = []
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize(dev)
    with ClockSampler(local_rank) as clk:
        for _ in range(steps):
            with torch.cuda.stream(stream):
                flush.zero_()  # L2 flush between steps, on the timed stream, before the step's start event
            s0 = torch.cuda.Event(enable_timing=True)
            s1 = torch.cuda.Event(enable_timing=True)
            s0.record(stream)
            step(True)
            s1.record(stream)
            step_ms.append((s0, s1))
        torch.cuda.synchronize(dev)
    if world > 1:
        dist.barrier()
    launches = sum(p.launches for p in plans) - launches0
    ms = [a.elapsed_time(b) for a, b in step_ms]
    ms_step = sum(ms) / len(ms)
    phase_ms = [sum(a.elapsed_time(b) for a, b in evs) / len(evs) for evs in ev_phase]
    if world > 1:
        t = torch.tensor([ms_step] + phase_ms, dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms_step, phase_ms = float(t[0]), [float(v) for v in t[1:]]

    # every output in input order (gathered at N > 1): its hash is the same at every N
    torch.cuda.synchronize(dev)
    digest = None
    if rank == 0:
        sc_list = [final[f"scores{k}"] for k in range(len(scores))] if sharded else scores
        h = hashlib.sha256()
        for s in sc_list:
            h.update(s.cpu().numpy().tobytes())
        if tb_plan is not None:
            tb_t, tl_t = (final["tb"], final["tl"]) if sharded else (tb_out, tb_len)
            cols = torch.arange(stride, device=dev)[None, :]
            valid = torch.where(cols < tl_t[:, None].long(), tb_t, torch.zeros_like(tb_t))
            h.update(tl_t.cpu().numpy().tobytes())
            h.update(valid.cpu().numpy().tobytes())
        digest = h.hexdigest()[:16]

    # HMM: each kernel's own time, alone (the step overlaps them); the forward's roofline uses it
    alone = {}
    if W["kind"] == "hmm":
        for k, nm in ((0, "k_forward_tc"), (1, "k_viterbi")):
            a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            reps = 3
            with torch.cuda.stream(stream):
                flush.zero_()
                a0.record(stream)
                for _ in range(reps):
                    plans[k].solve_batch(*dev_in, max_len_a=W["max_la"], max_len_b=0, out=scores[k], stream=stream)
                a1.record(stream)
            torch.cuda.synchronize(dev)
            alone[nm] = a0.elapsed_time(a1) / reps
        alone["vit_kernel"] = plans[1].last_variant  # k_viterbi16 (s16x2) or k_viterbi (int32 keys)
        a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(stream):
            a0.record(stream)
            tb_plan.traceback_into(0, n, tb_out, stride, tb_len, tb_co, stream=stream)
            a1.record(stream)
        torch.cuda.synchronize(dev)
        alone["k_viterbi_copy"] = a0.elapsed_time(a1)

    fixed = None
    intra = None
    nocl = None
    if name == "nussmid":   # NEXT 4 evidence: the same batch on the warp-per-problem batch kernel
        os.environ["DP_NUSS_NO_CLUSTER"] = "1"
        try:
            with make_plans(dp, W)[0] as pb:
                with torch.cuda.stream(stream):
                    pb.solve_batch(*dev_in, max_len_a=W["max_la"], out=scores[0], stream=stream)
                    f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    f0.record(stream)
                    for _ in range(3):
                        pb.solve_batch(*dev_in, max_len_a=W["max_la"], out=scores[0], stream=stream)
                    f1.record(stream)
                torch.cuda.synchronize(dev)
                nocl = round(f0.elapsed_time(f1) / 3, 4)
        finally:
            del os.environ["DP_NUSS_NO_CLUSTER"]
    if W["kind"] == "swshort":   # the hybrid's evidence: the same batch on the intra-task warp kernel
        os.environ["DP_SW_INTRA"] = "1"
        try:
            with make_plans(dp, W)[0] as pi:
                def both():
                    pi.solve_batch(*dev_in, max_len_a=W["max_la"], max_len_b=W["max_lb"], out=scores[0], stream=stream)
                    pi.traceback_into(0, n, tb_out, stride, tb_len, tb_co, stream=stream)
                with torch.cuda.stream(stream):
                    both()
                    f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    f0.record(stream)
                    for _ in range(3):
                        both()
                    f1.record(stream)
                torch.cuda.synchronize(dev)
                intra = round(f0.elapsed_time(f1) / 3, 4)
        finally:
            del os.environ["DP_SW_INTRA"]
    if W["kind"] == "diag":   # §4.7 evidence: the same batch with each candidate forced for every problem
        fixed = {}
        for a in dp.schedule_conditional(2, [((-1, -1), None, 0, 0)]):
            with dp.Plan(dp.DIAG_LCS, W["max_la"], W["max_lb"], alphabet_size=4, user_coeff=a) as pf:
                with torch.cuda.stream(stream):
                    pf.solve_batch(*dev_in, max_len_a=W["max_la"], max_len_b=W["max_lb"], out=scores[0], stream=stream)
                    f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    f0.record(stream)
                    for _ in range(3):
                        pf.solve_batch(*dev_in, max_len_a=W["max_la"], max_len_b=W["max_lb"], out=scores[0],
                                       stream=stream)
                    f1.record(stream)
                torch.cuda.synchronize(dev)
                fixed[str(tuple(a))] = round(f0.elapsed_time(f1) / 3, 4)

    e2e = e2e_host(W, plans, dev, stream, world, steps=max(1, min(steps, 5)))
    roof = roofline(W, name, phase_ms, alone, peaks())
    res = {
        "value": round(W["cells_total"] / (ms_step * 1e-3) / 1e9, 3) if (sharded or world == 1)
        else round(W["cells_local"] * world / (ms_step * 1e-3) / 1e9, 3),
        "unit": "GCUPS",
        "ms_per_step": round(ms_step, 4),
        "steps": steps, "warmup": warmup,
        "scaling": ("strong" if sharded else ("replicas" if world > 1 and name in ("nuss1", "nuss4") else
                                              ("weak" if world > 1 else "strong"))),
        "dtype": {"sw": "s16x2 (int16 lanes; score range plan-checked, else int32)",
                  "swa": ("s16x2 keys 4 v + code (int16 lanes; score range plan-checked, else int32)"
                          if W.get("variant") == "k_affine16" else "int32"), "swshort": "int32", "nuss": "int16 table, s16x2 max-plus (score <= n/2)",
                  "diag": "uint16 table / int32", "hmm": "f32 (forward; bf16x3 tensor-core split) + s16x2 (Viterbi: int16 lanes relative to the row max, exactness plan-checked, else int32)",
                  "phmm": "f32 (scaled linear space, per-lane power-of-two exponents)"}[W["kind"]],
        "config": {"workload": W["workload"], "config": name, "problems": W["n_total"], "problems_per_gpu": n,
                   "cells": W["cells_total"],
                   "l2": "flushed between steps (256 MiB write on the timed stream before each step's start event)",
                   "parallelism": (f"dp{world}: batch sharded, NCCL all-gather to input order" if sharded else
                                   (f"{world} replicas" if world > 1 else "1 GPU"))},
        "kernel_ms": round(phase_ms[0], 4),
        "phases_ms": {nm: round(v, 4) for nm, v in zip(phase_names, phase_ms)},
        "roofline": roof,
        "gpu_launches": int(launches),
        "result_sha256": digest,
        **({"alone_ms": {k: (round(v, 4) if isinstance(v, float) else v) for k, v in alone.items()}} if alone else {}),
        **({"batch_kernel_ms": nocl, "cluster_kernel_ms": round(phase_ms[0], 4)} if nocl else {}),
        **({"intra_task_ms": intra, "inter_task_ms": round(ms_step, 4)} if intra else {}),
        **({"fixed_schedule_ms": fixed, "conditional_schedule_ms": round(ms_step, 4)} if fixed else {}),
        "e2e": e2e,
        "clocks": clk.summary(),
    }
    if rank == 0 and world == 1 and not args.no_cpu:
        res["cpu_baseline"] = cpu_baseline(name, W)
    for p in plans:
        p.close()
    del dev_in, flush
    torch.cuda.empty_cache()
    return res


def roofline(W, name, phase_ms, alone, pk):
    """Roofline of the config's dominant kernel. `achieved` counts ALGORITHMIC work only (SURVEY.md
    §8(d)): max-plus lane-ops for the alignment sweeps, split evaluations for
    Nussinov, add-max for Viterbi, 2 S^2 flops per cell for the forward."""
    clock_hz = pk["sm_max_mhz"] * 1e6
    peak16 = MEASURED_UBENCH["viaddmnmx_s16x2"] * SMS * clock_hz
    peak32 = MEASURED_UBENCH["viaddmnmx_s32"] * SMS * clock_hz
    traffic = traffic_table()

    def alu(kernel, ops, ms, peak, note, units=1):
        ach = ops / (ms * 1e-3)
        t = traffic.get(kernel)
        return {"bound": "alu", "kernel": kernel, "achieved": round(ach / 1e12, 5), "peak": round(peak / 1e12, 4),
                "unit": "Tops/s", "frac": round(ach / peak, 4),
                "traffic": (round(t["bytes_per_launch"] * units) if t else None),
                **({"traffic_note": t.get("note", "")} if t else {}),
                "kernel_ms": round(ms, 4), "peak_source": note}

    if W["kind"] == "sw":
        ops = W["ops_local"]
        r = alu("k_sw16", ops, phase_ms[0], peak16,
                "ubench_r01 VIADDMNMX.S16x2 128 lane-ops/clk/SM x 148 SMs x sm_max_mhz (3 max-plus ops per cell)",
                units=W["cells_local"] / 6.5536e9)
        r["frac_vs_int32_peak"] = round(ops / (phase_ms[0] * 1e-3) / peak32, 4)
        r["traceback_ms"] = round(phase_ms[1], 4)
        return r
    if W["kind"] == "swshort":
        r = alu("k_sw_inter", W["ops_local"], phase_ms[0], peak32,
                "ubench_r01 VIADDMNMX s32 64 lane-ops/clk/SM x 148 SMs x sm_max_mhz (3 max-plus ops per cell; "
                "kernel time includes the 3 small length-sort launches)")
        r["traceback_ms"] = round(phase_ms[1], 4)
        return r
    if W["kind"] == "swa":
        if W.get("variant") == "k_affine16":
            r = alu("k_affine16", W["ops_local"], phase_ms[0], peak16,
                    "ubench_r01 VIADDMNMX.S16x2 128 lane-ops/clk/SM x 148 SMs x sm_max_mhz (6 max-plus ops per cell)")
            r["frac_vs_int32_peak"] = round(W["ops_local"] / (phase_ms[0] * 1e-3) / peak32, 4)
        else:
            r = alu("k_align_affine", W["ops_local"], phase_ms[0], peak32,
                    "ubench_r01 VIADDMNMX s32 64 lane-ops/clk/SM x 148 SMs x sm_max_mhz (6 int32 ops per cell)")
        r["traceback_ms"] = round(phase_ms[1], 4)
        return r
    if W["kind"] == "diag":
        return alu("k_diag", W["ops_local"], phase_ms[0], peak32,
                   "ubench_r01 VIADDMNMX s32 64 lane-ops/clk/SM x 148 SMs x sm_max_mhz (3 int ops per cell)")
    if W["kind"] == "nuss":
        if name == "nuss1":  # one problem, one SM: latency-bound; the fraction is of ONE SM's peak (§8(d) D1)
            one_sm = MEASURED_UBENCH["viaddmnmx_s16x2"] * clock_hz
            r = alu("k_nuss_small", W["inner_local"], phase_ms[0], one_sm,
                    "ubench_r01 VIADDMNMX.S16x2 128 lane-ops/clk x ONE SM x sm_max_mhz (one split evaluation = one "
                    "max-plus); latency-bound: 64 dependent partitions")
            r["bound"] = "latency"
            return r
        kname = {"nuss4": "k_nuss_grid2", "nussmid": "k_nuss_cluster"}.get(name, "k_nuss_batch")
        return alu(kname, W["inner_local"], phase_ms[0], peak16,
                   "ubench_r01 VIADDMNMX.S16x2 x 148 SMs x sm_max_mhz (one split evaluation = one max-plus)")
    if W["kind"] == "phmm":
        # forward: per (position j, index i) nine transition products and two emission products (M, I)
        # = 11 fp32 FMA-pipe lane-ops; roofline = the FFMA SIMT peak
        peakf = MEASURED_UBENCH["ffma"] * SMS * clock_hz
        r = alu("k_phmm_forward", 11 * W["inner_local"], phase_ms[0], peakf,
                "ubench_r01 FFMA 128 lane-ops/clk/SM x 148 SMs x sm_max_mhz (11 FMA-pipe ops per position and "
                "residue: 9 transition products + 2 emissions)")
        r["unit"] = "Tops/s (fp32 FMA pipe)"
        return r
    # HMM: Viterbi (max-plus, SIMT, the step's critical path) and the tcgen05 forward on its own time
    vk = alone.get("vit_kernel", "k_viterbi")
    vit_ms = alone.get("k_viterbi", phase_ms[1])
    if vk == "k_viterbi16":
        vit = alu(vk, W["inner_local"], vit_ms, peak16,
                  "ubench_r01 VIADDMNMX.S16x2 128 lane-ops/clk/SM x 148 SMs x sm_max_mhz (one 16-bit add-max per "
                  "(p, s, t)); the kernel time includes the fused path walk (argmax recovery)")
    else:
        vit = alu(vk, W["inner_local"], vit_ms, peak32,
                  "ubench_r01 VIADDMNMX s32 64 lane-ops/clk/SM x 148 SMs x sm_max_mhz (one add-max per (p, s, t)); "
                  "the kernel time includes the fused path walk")
    vit["kernel_ms_in_step"] = round(phase_ms[1], 4)
    fl = 2 * W["inner_local"]
    fw_ms = alone.get("k_forward_tc", phase_ms[0])
    tc3 = pk.get("bf16_tflops", 1685.9) * 1e12 / 3
    t = traffic.get("k_forward_tc")
    vit["forward_tc"] = {
        "bound": "tensor", "kernel": "k_forward_tc", "achieved": round(fl / (fw_ms * 1e-3) / 1e12, 3),
        "peak": round(tc3 / 1e12, 1), "unit": "TFLOP/s", "frac": round(fl / (fw_ms * 1e-3) / tc3, 4),
        "traffic": (round(t["bytes_per_launch"]) if t else None), "kernel_ms": round(fw_ms, 4),
        "peak_source": "MEASURED_PEAKS.json bf16_tflops (burst) / 3: the fp32 product is computed as three bf16 "
                       "MMAs (hi x hi, hi x lo, lo x hi); algorithmic flops 2 S^2 per cell; kernel timed alone",
        # SURVEY 8(d) D3's SIMT roofline: the same flops against the FFMA peak (2 flops per lane-op)
        "frac_vs_ffma_peak": round(fl / (fw_ms * 1e-3) / (2 * MEASURED_UBENCH["ffma"] * SMS * pk["sm_max_mhz"] * 1e6), 4)}
    return vit


def e2e_host(W, plans, dev, stream, world, steps):
    """Same metric through dp_solve_batch_host: pinned host inputs, H2D, solve, traceback, D2H, per
    rank on its shard (every rank returns its shard's results to host memory)."""
    import torch

    def pin(x):
        return torch.from_numpy(np.ascontiguousarray(x)).pin_memory().numpy()

    a_cat, a_off = pin(W["a_cat"]), pin(W["a_off"])
    b_cat = pin(W["b_cat"]) if "b_cat" in W else None
    b_off = pin(W["b_off"]) if "b_off" in W else None
    n, stride = len(W["a_off"]) - 1, W["tb_stride"] or 0
    fwd_like = W["kind"] in ("hmm", "phmm")
    outs = []
    for k, p in enumerate(plans):
        sc = pin(np.empty(n, np.float32 if (fwd_like and k == 0) else np.int32))
        tb = pin(np.empty((n, stride), np.uint8)) if p.want_traceback else None
        tl = pin(np.empty(n, np.int32)) if p.want_traceback else None
        tc = pin(np.empty((n, 4), np.int32)) if (p.want_traceback and W["kind"] in ("sw", "swa", "swshort")) else None
        outs.append((sc, tb, tl, tc))
    h2d = (a_cat.nbytes + a_off.nbytes + (b_cat.nbytes + b_off.nbytes if b_cat is not None else 0)) * len(plans)
    d2h = sum(o[0].nbytes + (o[1].nbytes + o[2].nbytes if o[1] is not None else 0) +
              (o[3].nbytes if o[3] is not None else 0) for o in outs)
    # HMM: the forward's host call on a high-priority stream, as in the device-timed step
    streams = ([torch.cuda.Stream(device=dev, priority=-1)] if len(plans) > 1 else [stream]) + \
        [torch.cuda.Stream(device=dev) for _ in plans[1:]]
    errors = []

    def run(k):
        try:
            torch.cuda.set_device(dev)
            sc, tb, tl, tc = outs[k]
            plans[k].solve_batch_host_into(a_cat, a_off, b_cat, b_off, sc, tb, stride, tl, tc, stream=streams[k])
        except Exception as ex:  # re-raised below: a failed call must not be timed as work done
            errors.append(ex)

    def one():
        # several plans over the same inputs (HMM forward + Viterbi) are independent calls: a user
        # runs them from two host threads on two streams (ctypes releases the GIL)
        if len(plans) == 1:
            run(0)
        else:
            ths = [threading.Thread(target=run, args=(k,)) for k in range(len(plans))]
            for t in ths:
                t.start()
            for t in ths:
                t.join()
        if errors:
            raise errors[0]

    one()
    torch.cuda.synchronize(dev)
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    t0 = time.perf_counter()
    e0.record(stream)
    for _ in range(steps):
        one()
    e1.record(stream)
    torch.cuda.synchronize(dev)
    wall = (time.perf_counter() - t0) * 1e3 / steps
    ms = max(e0.elapsed_time(e1) / steps, 0.0)
    if world > 1:
        import torch.distributed as dist
        t = torch.tensor([ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t[0])
    cells = W["cells_local"] * world
    return {"value": round(cells / (ms * 1e-3) / 1e9, 3), "unit": "GCUPS", "ms_per_step": round(ms, 3),
            "wall_ms_per_step": round(wall, 3),
            "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(d2h),
            "api": "dp_solve_batch_host (pinned host buffers; H2D + solve + traceback + D2H), per rank shard"}


# ----------------------------------------------------------------------------- oracle (CPU)
def host_cores():
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


def oracle_sample(config, W):
    """Times the oracle as it stands on a bounded sample (~5-20 s of CPU work); returns
    (cells/s of the config's own workload, sample text, cores)."""
    import oracle
    cores = host_cores()
    if config == "sw":
        k = 4000
        a_cat, a_off, b_cat, b_off = dpgen.config2_protein_pairs(k)
        sig = dpgen.blosum62()
        t = time.perf_counter()
        oracle.sw_batch(a_cat, a_off, b_cat, b_off, sig, dpgen.SW_GAP, threads=cores)
        oracle.sw_traceback_batch(a_cat, a_off, b_cat, b_off, sig, dpgen.SW_GAP, 513, threads=cores)
        dt = time.perf_counter() - t
        return k * 65536 / dt, f"first {k} pairs of config 2 (scores + canonical tracebacks)", cores
    if config == "swshort":
        k = 60000
        a_cat, a_off, b_cat, b_off = dpgen.short_protein_pairs(k)
        sig = dpgen.blosum62()
        t = time.perf_counter()
        oracle.sw_batch(a_cat, a_off, b_cat, b_off, sig, dpgen.SW_GAP, threads=cores)
        oracle.sw_traceback_batch(a_cat, a_off, b_cat, b_off, sig, dpgen.SW_GAP, 129, threads=cores)
        dt = time.perf_counter() - t
        return int((np.diff(a_off) * np.diff(b_off)).sum()) / dt, \
            f"first {k} pairs of the short-pair workload (scores + canonical tracebacks)", cores
    if config == "swa":
        k = 1500
        a_cat, a_off, b_cat, b_off = dpgen.config2_protein_pairs(k)
        sig = dpgen.blosum62()
        go, ge = dpgen.SW_GAP_OPEN, dpgen.SW_GAP_EXTEND
        t = time.perf_counter()
        oracle.sw_affine_batch(a_cat, a_off, b_cat, b_off, sig, go, ge, threads=cores)
        oracle.sw_affine_traceback_batch(a_cat, a_off, b_cat, b_off, sig, go, ge, 513, threads=cores)
        dt = time.perf_counter() - t
        return k * 65536 / dt, f"first {k} pairs of config 2, affine gaps (scores + canonical tracebacks)", cores
    if config == "nuss1":
        x = dpgen.config1_rna64()
        reps = 200
        t = time.perf_counter()
        for _ in range(reps):
            oracle.nussinov_traceback(x, dpgen.rna_pair_mask(), 3)
        dt = time.perf_counter() - t
        return reps * 2016 / dt, f"config 1 x{reps} repetitions (score + traceback), 1 core", 1
    if config == "diag":
        k = 150
        a_cat, a_off, b_cat, b_off = dpgen.diag_pairs(k)
        t = time.perf_counter()
        oracle.lcsubstr_batch(a_cat, a_off, b_cat, b_off, threads=cores)
        dt = time.perf_counter() - t
        return int((np.diff(a_off) * np.diff(b_off)).sum()) / dt, f"first {k} pairs of the diag workload", cores
    if config == "nuss4":
        # the n = 8192 oracle takes ~1 h single-threaded (tests/golden/config4.json records
        # it); time the config-4 sequence's first 2048 nt and extrapolate by split evaluations
        x = dpgen.config4_rna8192()[:2048]
        t = time.perf_counter()
        oracle.nussinov_traceback(x, dpgen.rna_pair_mask(), 3)
        dt = time.perf_counter() - t
        ev = lambda n: n * (n - 1) * (n - 2) / 6
        dt8 = dt * ev(8192) / ev(2048)
        return 8192 * 8191 / 2 / dt8, (f"first 2048 nt of config 4 (score + traceback, 1 core) in {dt:.1f} s, "
                                       f"extrapolated by split evaluations to n = 8192 ({dt8:.0f} s)"), 1
    if config == "nussmid":
        cat, off = dpgen.mid_rna_batch()
        k = 3
        t = time.perf_counter()
        for q in range(k):
            oracle.nussinov_traceback(cat[off[q]:off[q + 1]], dpgen.rna_pair_mask(), 3)
        dt = time.perf_counter() - t
        lens = np.diff(off)[:k]
        return int((lens * (lens - 1) // 2).sum()) / dt, f"first {k} problems of the nussmid batch (score + traceback, 1 core)", 1
    if config == "nuss5":
        ids = dpgen.config5_sample_ids(k=2000)
        cat, off = dpgen.config5_rna_batch(ids=ids)
        lens = np.diff(off)
        t = time.perf_counter()
        oracle.nussinov_batch(cat, off, dpgen.rna_pair_mask(), 3, threads=cores)
        dt = time.perf_counter() - t
        cells = int((lens * (lens - 1) // 2).sum())
        return cells / dt, f"{len(ids)} sequences of the fixed config-5 subset (seed +7), scores only", cores
    if config == "phmm":
        d = dpgen.profile_hmm_workload(n_seqs=200)
        t = time.perf_counter()
        oracle.profile_forward_batch(d["cat"], d["off"], d["L"], **d["model64"], threads=cores)
        dt = time.perf_counter() - t
        return 3 * d["L"] * int(np.diff(d["off"]).sum()) / dt, "first 200 sequences of the profile-HMM workload", cores
    d = dpgen.config3_hmm(n_seqs=200)
    k = 200
    seqs = d["seqs"][:k]
    off = np.arange(k + 1, dtype=np.int64) * seqs.shape[1]
    t = time.perf_counter()
    oracle.forward_batch(seqs.reshape(-1), off, *(d[q].astype(np.float64) for q in ("pi", "A", "E")), threads=cores)
    oracle.viterbi_batch(seqs.reshape(-1), off, d["lpi"], d["lA"], d["lE"], threads=cores)
    dt = time.perf_counter() - t
    return 2 * k * 64 * 1000 / dt, f"first {k} sequences of config 3 (forward + Viterbi)", cores


def cpu_baseline(config, W):
    v, sample, cores = oracle_sample(config, W)
    return {"value": round(v / 1e9, 6), "unit": "GCUPS", "cores": cores, "kind": "oracle", "sample": sample}


def run_reference(args, rank, world):
    """--impl reference: the oracle as it stands on the host cores, bounded samples per step."""
    if rank != 0:
        return None
    vals = []
    sample = cores = None
    for k in range(args.warmup + args.steps):
        v, sample, cores = oracle_sample(args.config, None)
        if k >= args.warmup:
            vals.append(v)
    val = sum(vals) / len(vals)
    wl = {"sw": "BASELINE config 2: 100k protein pairs x 256 (uniform 20 aa), Smith-Waterman, BLOSUM62, linear gap 4, "
                "with tracebacks"}.get(args.config, f"config {args.config}")
    return {
        "impl": "reference", "metric": METRIC,
        "value": round(val / 1e9, 6), "unit": "GCUPS", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
        "dtype": "int64 (oracle)", "data": "synthetic (seeded, dpgen)",
        "config": {"workload": wl, "config": args.config},
        "cpu_baseline": {"value": round(val / 1e9, 6), "unit": "GCUPS", "cores": cores, "kind": "oracle",
                         "sample": sample},
        "e2e": {"value": round(val / 1e9, 6), "unit": "GCUPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }


DEFAULT_STEPS = {"sw": 60, "swa": 20, "swshort": 30, "nussmid": 20, "hmm": 30, "nuss1": 200, "nuss4": 15, "nuss5": 2, "diag": 25, "phmm": 20}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=None,
                    help="timed steps of the headline (default per config: ~0.15 s, so the clock sampler sees it)")
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="sw", choices=ALL_CONFIGS)
    ap.add_argument("--only", action="store_true", help="headline config only (no `configs` block)")
    ap.add_argument("--configs", default=None, help="comma list for the `configs` block (default: all others)")
    ap.add_argument("--scaling", default="strong", choices=["strong", "weak"])
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline legs")
    args = ap.parse_args()
    if args.steps is None:
        args.steps = DEFAULT_STEPS[args.config] if args.impl == "ours" else 3
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        # self-launch one rank per GPU (NCCL_DEBUG=INFO makes the communicator's rank count visible)
        env = dict(os.environ, NCCL_DEBUG=os.environ.get("NCCL_DEBUG", "INFO"))
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
               "--master-addr=127.0.0.1", f"--master-port={29500 + os.getpid() % 1000}", __file__] + sys.argv[1:]
        sys.exit(subprocess.call(cmd, env=env))
    if args.impl == "reference":
        res = run_reference(args, rank, world)
        if res is not None:
            print(json.dumps(res), flush=True)
        return
    import torch
    # DP_BENCH_BACKEND=gloo (tests only): several ranks on fewer GPUs, to exercise the N > 1 shard /
    # gather path where only one GPU is available; the product path is NCCL, one rank per GPU
    backend = os.environ.get("DP_BENCH_BACKEND", "nccl")
    if backend != "nccl":
        local_rank = local_rank % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local_rank)
    if world > 1:
        import torch.distributed as dist
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
        else:
            dist.init_process_group(backend)
    head = run_config(args.config, args, rank, world, local_rank, args.steps, args.warmup, True)
    res = {"metric": METRIC, "value": head.pop("value"), "unit": "GCUPS", "n_gpus": world, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": head.pop("ms_per_step"), "higher_is_better": True,
           "scaling": head.pop("scaling"), "vs_baseline": None, "dtype": head.pop("dtype"),
           "data": "synthetic (seeded, dpgen; SURVEY §8(d) recipes)"}
    head.pop("steps", None)
    head.pop("warmup", None)
    res.update(head)
    if not args.only:
        names = args.configs.split(",") if args.configs else [c for c in ALL_CONFIGS if c != args.config]
        if world > 1:
            names = [c for c in names if c in SHARDED]
        block = {}
        for c in names:
            st = min(DEFAULT_STEPS[c], args.steps)
            try:
                block[c] = run_config(c, args, rank, world, local_rank, st, min(args.warmup, 3), False)
            except Exception as ex:  # a config that fails is reported, never silently dropped
                block[c] = {"error": f"{type(ex).__name__}: {ex}"[:300]}
        res["configs"] = block
    if rank == 0:
        print(json.dumps(res), flush=True)
    if world > 1:
        import torch.distributed as dist
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
