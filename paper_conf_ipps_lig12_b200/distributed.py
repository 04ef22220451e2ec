"""H9 — cross-GPU reduction of one check's summary.

The parameter space shards by seed (rank r takes seeds r, r + world, ...; or, in
weak-scaling runs, its own seed range), so evaluation needs no communication.
Only the first-counterexample keys (int64[11], all_reduce MIN) and the counts
(int64[16], all_reduce SUM) cross the interconnect - NCCL over NVLink on the GPU
box, gloo in the CPU tests.  Records stay on their rank; `merge_records` merges
the per-rank lists on the host (canonical key order is preserved because keys
embed (launch, seed_idx, kernel, kind, round), X16).
"""
from __future__ import annotations

import heapq
from typing import Iterable, List, Sequence

INT64_MAX = 2 ** 63 - 1


def reduce_summary(first_key, counts, group=None):
    """In place: first_key <- MIN over ranks, counts <- SUM over ranks (torch tensors)."""
    import torch.distributed as dist
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(first_key, op=dist.ReduceOp.MIN, group=group)
        dist.all_reduce(counts, op=dist.ReduceOp.SUM, group=group)
    return first_key, counts


def merge_records(per_rank: Sequence[Iterable[tuple]]) -> List[tuple]:
    """Merge per-rank record lists (each already in canonical order) by (key, array, addr, tid_a, tid_b)."""
    def order(r):
        # REC_FIELDS = key, count, kind, launch, seed_idx, kernel, round, site, array, addr, tid_a, tid_b, ...
        return (r[0], r[8], r[9], r[10], r[11])
    return list(heapq.merge(*[list(p) for p in per_rank], key=order))


def first_witness(first_key: int):
    """Decode the first-witness launch / seed index from a key (X16); None if no failure."""
    if first_key >= INT64_MAX:
        return None
    return {"launch": first_key >> 45, "seed_idx": (first_key >> 24) & 0x1FFFFF, "kernel": (first_key >> 20) & 0xF,
            "kind": (first_key >> 16) & 0xF, "round": first_key & 0xFFFF}


def greedy_assignment(costs: Sequence[float], n_seeds: Sequence[int], world: int, chunk: int = 0):
    """where seeds are few per launch (C4's exhaustive 0/1 sets, one-seed
    runs), round-robin seed shards leave ranks idle; instead the (launch, seed) instances
    are assigned greedily by cost (longest processing time first: items sorted by cost, each
    to the least-loaded rank).  costs[l] = cost of one (launch l, seed) instance (e.g.
    threads x rounds x ops), n_seeds[l] = its seeds.  Items are (launch, seed range) chunks
    of `chunk` seeds (default: enough to give every rank several items).  Returns, per rank,
    a list of (launch, seed0, seed1) in launch order - each becomes a sub-space whose
    pg_space.key_launch0 / key_seed0 put its records at their global keys."""
    if world < 1:
        raise ValueError("world >= 1")
    total = sum(int(s) for s in n_seeds)
    chunk = chunk or max(1, total // (8 * world))
    items = []
    for l, (c, ns) in enumerate(zip(costs, n_seeds)):
        for a in range(0, int(ns), chunk):
            b = min(int(ns), a + chunk)
            items.append((float(c) * (b - a), l, a, b))
    items.sort(key=lambda x: (-x[0], x[1], x[2]))
    load = [0.0] * world
    out = [[] for _ in range(world)]
    for c, l, a, b in items:
        r = min(range(world), key=lambda i: (load[i], i))
        load[r] += c
        out[r].append((l, a, b))
    for r in range(world):   # merge adjacent seed ranges of a launch, launch order
        merged = []
        for l, a, b in sorted(out[r]):
            if merged and merged[-1][0] == l and merged[-1][2] == a:
                merged[-1] = (l, merged[-1][1], b)
            else:
                merged.append((l, a, b))
        out[r] = merged
    return out
